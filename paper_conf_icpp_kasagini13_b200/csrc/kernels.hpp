// kernels.hpp — launchers of the sm_100a kernels (libperm internals).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "plan.hpp"

namespace perm {

// Registers max dynamic shared memory for every kernel instantiation the plan uses.
cudaError_t prepare_kernels(HostPlan& P);   // also sets persistent grid sizes

// All three phases in one CTA (n <= 2^15): a -> smem -> R1, R2 (columns), R3 -> b.
cudaError_t launch_fused(const HostPlan& P, const uint32_t* const sched[3], const uint32_t* a,
                         uint32_t* b, cudaStream_t s);

// Cluster path (n = 2^15..2^18): one launch of one cluster of P.cluster blocks; all three
// phases in distributed shared memory, the column phase's transposes as block exchanges.
cudaError_t launch_cluster(const HostPlan& P, const uint32_t* const sched[3], const uint32_t* a,
                           uint32_t* b, cudaStream_t s, unsigned long long* trace = nullptr);

// One row pass (pass index f in 0..2) of the 3- or 5-pass pipeline.
// `trace`: optional device buffer of 16 %globaltimer stamps per CTA (nullptr = off).
// `map`: the X1 / X2 tensor map when the pass is a TLC ring pass (layout 5) with chunked output.
cudaError_t launch_row_pass(const HostPlan& P, int f, const uint32_t* sched, const uint32_t* in,
                            uint32_t* out, cudaStream_t s, bool pdl,
                            unsigned long long* trace = nullptr, const CUtensorMap* map = nullptr);

// TLC layout: tensor maps of the intermediates (maps[0]: X1 for pass 1's 3-D
// stores, maps[1]: X2 for pass 2's 4-D stores) and one pass launch.
cudaError_t make_tlc_maps(const HostPlan& P, uint32_t* x1, uint32_t* x2, CUtensorMap* maps);
cudaError_t launch_tlc_pass(const HostPlan& P, int f, const CUtensorMap* maps, const uint32_t* sched,
                            const uint32_t* in, uint32_t* out, cudaStream_t s, bool pdl,
                            unsigned long long* trace = nullptr);

// TLC layout, square views: the three passes in one persistent launch.
cudaError_t launch_tlc_fused(const HostPlan& P, const CUtensorMap* maps, const uint32_t* const sched[3],
                             const uint32_t* a, uint32_t* x1, uint32_t* x2, uint32_t* b,
                             unsigned long long* sync, cudaStream_t s,
                             unsigned long long* trace = nullptr);

// out (cols x rows) = transpose of in (rows x cols), 32 x 32 tiles (§V).
cudaError_t launch_transpose(const uint32_t* in, uint32_t* out, int64_t rows, int64_t cols,
                             cudaStream_t s, bool pdl);

// Comparators and a plain vector copy.
cudaError_t launch_scatter(const int32_t* p, const void* a, void* b, int64_t n, int eb,
                           cudaStream_t s);
cudaError_t launch_gather(const int32_t* q, const void* a, void* b, int64_t n, int eb,
                          cudaStream_t s);
cudaError_t launch_block_gather(const int32_t* qb, const void* a, void* b, int64_t n_words,
                                cudaStream_t s);
cudaError_t launch_copy(const uint32_t* a, uint32_t* b, int64_t n, cudaStream_t s);

}  // namespace perm
