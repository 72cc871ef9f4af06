// gplan.hpp — GPU colourings of the offline plan builder (gplan.cu).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

namespace perm {

struct GpuPlanStats {
    int32_t levels = 0;          // Euler-split levels run (log2 of the degree, summed over calls)
    int32_t jump_rounds = 0;     // pointer-jumping rounds over the reduced (ruler) lists
    int64_t reduced_nodes = 0;   // reduced-list sizes, summed over levels
};

// Row-level colouring (Thm 6): kappa[x] in [0, c) for the
// c-regular multigraph source row x >> logc -> destination row p[x] >> logc,
// on the current device. p, kappa: host arrays of n entries.
cudaError_t gpu_row_colour(const int32_t* p_host, int64_t n, int logc, uint16_t* kappa_host,
                           GpuPlanStats* st);

// Bank-level colourings (L531-L533) of E / B independent blocks of B = 2^logB
// elements: edge e joins (block, keyU[e] & 31) to (block, keyV[e] & 31); keyU
// and keyV are bijections onto [0, B) within each block (keyU == nullptr: keyU[e] =
// e mod B, the line order). col[e] in [0, B/32).
cudaError_t gpu_bank_colour(const uint16_t* keyU_host, const uint16_t* keyV_host, int64_t E, int logB,
                            uint16_t* col_host, GpuPlanStats* st);

// Bank colouring + W64 packing of one phase's per-line schedules (plan.hpp
// entry_pos32: W64 or dense) on the device: phi = Phi per element in line order (n
// entries, lines of 2^logL); words: host array of (n/32)*(dense ? E : 2*w64) u32.
cudaError_t gpu_line_schedules(const uint16_t* phi_host, int64_t n, int logL, int E, int epw, int w64,
                               int dense, uint32_t* words_host, GpuPlanStats* st);

}  // namespace perm
