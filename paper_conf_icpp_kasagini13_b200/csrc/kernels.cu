// kernels.cu — sm_100a kernels of libperm.
//
// The data-parallel hot path of the scheduled offline permutation
// (§V-§VII): row-wise permutations driven by a bank-conflict-free
// schedule (Lemma 7) and the transposes that turn a column-wise
// permutation into a row-wise one (Lemma 5/8, L409-L423, L533).
//
// B200 design:
//  * a CTA owns h whole lines in shared memory (one line = one DMM block of
//    the paper); global traffic is 128-bit and coalesced, staged through
//    shared memory whose line stride is padded so that the cross-line
//    accesses of the tiled layouts are also conflict-free (the padded
//    stride plays the role of the paper's diagonal arrangement, Fig. 4);
//  * the permute hop is done IN PLACE with register staging: every thread
//    reads its EPT sources sm[32*sigma + lane] (bank = lane), the CTA
//    synchronises, then every thread writes its destinations sm[t] (the 32
//    t of a warp-round are in 32 distinct banks). This halves shared memory
//    versus the paper's separate A_i / B_i arrays (L523);
//  * schedule entries are bit-packed (2*log2(L) - 5 bits, not the paper's
//    2 x 16-bit shorts, L699) and decoded with two warp shuffles;
//  * passes are chained with programmatic dependent launch: a pass
//    prefetches its schedule into L2 before griddepcontrol.wait, so the
//    schedule stream overlaps the previous pass.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstring>
#include <cstdlib>

#include "kernels.hpp"

namespace perm {

namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;

__host__ __device__ constexpr int cilog2(int v) { return v <= 1 ? 0 : 1 + cilog2(v >> 1); }

__device__ __forceinline__ void pdl_wait() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
}
__device__ __forceinline__ void pdl_launch_dependents() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void prefetch_l2(const void* p) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}
// polling wait with a sleep between probes: for a lone thread that waits for a long time
// (it stops competing for issue slots with the warps doing the work on its SM sub-partition)
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}" : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait_sleepy(uint64_t* bar, uint32_t parity, unsigned ns) {
    while (!mbar_test(bar, parity)) __nanosleep(ns);
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
// TMA 1-D bulk copy global -> shared, completion counted on an mbarrier
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}
// TMA 1-D bulk copy shared -> global (bulk group)
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
                 "r"(smem_u32(src)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void prefetch_l2_bulk(const void* p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read1() {
    asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// L2 eviction-priority policies (createpolicy) and a read-only load carrying one
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint32_t ld_nc_hint(const uint32_t* p, uint64_t pol) {
    uint32_t v;
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}

// intermediates X1 / X2 are re-read by the next pass: stored with an evict_last L2 policy
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, const void* src, int c0, int c1, int c2) {
    const uint64_t pol = policy_evict_last();
    asm volatile(
        "cp.async.bulk.tensor.3d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%2, %3, %4}], [%1], %5;" ::"l"(
            reinterpret_cast<uint64_t>(map)),
        "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2), "l"(pol)
        : "memory");
}

// streaming 128-bit load of data that is not written by this kernel
__device__ __forceinline__ uint4 ld_nc_v4(const uint32_t* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}
__device__ __forceinline__ void st_v4(uint32_t* p, uint4 v) {
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
                 "r"(v.w)
                 : "memory");
}

// ------------------------------------------------------------------ permute hop

// In-place permutation of the lines resident in shared memory. Warp-round q
// (0 <= q < h*L/32) of this CTA is line q >> (logL-5), round q & (L/32 - 1);
// warp w handles q = w + W*m for m < EPT. addr(l, pos) maps (line, position)
// to a shared-memory word: ROWS -> l*Ls + pos, COLS -> pos*Ls + l.
template <bool SMEM>
__device__ __forceinline__ uint2 sched_load64(const uint2* p) {
    if constexpr (SMEM) return *p;
    else return __ldg(p);
}
template <bool SMEM>
__device__ __forceinline__ uint32_t sched_load32(const uint32_t* p) {
    if constexpr (SMEM) return *p;
    else return __ldg(p);
}

// Entry of warp-round q for this lane, W64 or dense format (plan.hpp PhaseGeom).
// W64: 64-bit word q*w64 + lane/epw, shift E*(lane % epw). Dense: round q = E
// u32 words, lane's entry at bit lane*E (two loads + funnel shift; the second
// load repeats the first when the entry does not straddle).
struct SchedDec {
    int dense, E, w64, wsel, sh, dwo, dwo2, dbo;
    uint32_t mask;
    __device__ __forceinline__ SchedDec(int dense_, int E_, int epw, int w64_, int lane)
        : dense(dense_), E(E_), w64(w64_) {
        wsel = lane / epw;
        sh = E * (lane - wsel * epw);
        const int bit = lane * E;
        dwo = bit >> 5;
        dbo = bit & 31;
        dwo2 = dwo + ((dbo + E > 32) ? 1 : 0);
        mask = (1u << E) - 1u;
    }
    template <bool SMEM>
    __device__ __forceinline__ uint32_t get(const uint32_t* sched, int q) const {
        if (dense) {
            const uint32_t* p = sched + q * E;
            const uint32_t lo = sched_load32<SMEM>(p + dwo), hi = sched_load32<SMEM>(p + dwo2);
            return (uint32_t)((((uint64_t)hi << 32) | lo) >> dbo) & mask;
        }
        const uint2 wd = sched_load64<SMEM>(reinterpret_cast<const uint2*>(sched) + q * w64 + wsel);
        return (uint32_t)((((uint64_t)wd.y << 32) | wd.x) >> sh) & mask;
    }
};

// In-place permutation of the lines resident in shared memory. Warp-round q
// (0 <= q < h*L/32) of this CTA is line q >> (logL-5), round q & (L/32 - 1);
// warp w handles q = w + W*m for m < EPT. addr(l, pos) maps (line, position)
// to a shared-memory word: ROWS -> l*Ls + pos, COLS -> pos*Ls + l.
// Schedule in the W64 format (plan.hpp): lane x reads 64-bit word x/epw of the
// round and shifts by E*(x % epw): one load, no shuffles. The destination
// addresses decoded in the read hop stay in registers (two 16-bit addresses
// per register) for the write hop, so the schedule is read once.
template <int EPT, bool COLS, bool SCHED_SMEM = false>
__device__ __forceinline__ void permute_lines(uint32_t* sm, const uint32_t* __restrict__ sched,
                                              int logL, int E, int epw, int w64, int Ls, int dense = 0) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, W = blockDim.x >> 5;
    const int logR = logL - 5;                      // log2(rounds per line)
    const SchedDec dec(dense, E, epw, w64, lane);
    const uint32_t tmask = (1u << logL) - 1u;
    // Up to 32 elements per thread the decoded destinations stay in registers
    // (two 16-bit addresses per register); beyond that they are re-decoded in
    // the write hop to stay within 128 registers.
    constexpr bool KEEP = EPT <= 32;
    uint32_t v[EPT];
    uint32_t ta[KEEP ? (EPT + 1) / 2 : 1];
    // read hop: v[m] = line[32*sigma + lane]   (bank = lane + const: conflict-free)
#pragma unroll
    for (int m = 0; m < EPT; ++m) {
        const uint32_t e = dec.get<SCHED_SMEM>(sched, warp + W * m);
        const int l = (warp + W * m) >> logR;
        const int s = (int)((e >> logL) << 5) + lane;
        v[m] = COLS ? sm[s * Ls + l] : sm[l * Ls + s];
        if constexpr (KEEP) {
            const int t = (int)(e & tmask);
            const uint32_t ad = COLS ? (uint32_t)(t * Ls + l) : (uint32_t)(l * Ls + t);
            if (m & 1) ta[m >> 1] |= ad << 16;
            else ta[m >> 1] = ad;
        }
    }
    __syncthreads();
    // write hop: line[t] = v[m]   (the 32 t of a warp-round hit 32 distinct banks)
    if constexpr (KEEP) {
#pragma unroll
        for (int m = 0; m < EPT; ++m) sm[(ta[m >> 1] >> ((m & 1) * 16)) & 0xFFFFu] = v[m];
    } else {
        const int warp2 = __shfl_sync(kFull, warp, 0);   // not CSE-able: re-derive addresses
#pragma unroll
        for (int m = 0; m < EPT; ++m) {
            const uint32_t e = dec.get<SCHED_SMEM>(sched, warp2 + W * m);
            const int l = (warp2 + W * m) >> logR;
            const int t = (int)(e & tmask);
            if (COLS) sm[t * Ls + l] = v[m];
            else      sm[l * Ls + t] = v[m];
        }
    }
    __syncthreads();
}

// ------------------------------------------------------------------ fused (n <= 2^15)

struct FusedArgs {
    const uint32_t* in;
    uint32_t* out;
    const uint32_t* sched[3];
    int logr, logc, Ls, E[3], epw[3], w64[3];
};

// PAPER.md Thm 9: row-wise, column-wise, row-wise — all inside one CTA. The
// r x c matrix sits in shared memory with an odd row stride Ls = c + 1, so
// element (i, j) is in bank (i + j) mod 32: rows AND columns are conflict-free,
// exactly the property of the diagonal arrangement (Fig. 4). The column
// phase therefore needs no transpose at all.
template <int EPT>
__global__ void __launch_bounds__(512, 1) fused_kernel(const FusedArgs a) {
    extern __shared__ __align__(16) uint32_t sm[];
    const int T = blockDim.x, tid = threadIdx.x;
    const int n = 1 << (a.logr + a.logc);
    const int cmask = (1 << a.logc) - 1;
    for (int e = tid; e < n; e += T) sm[(e >> a.logc) * a.Ls + (e & cmask)] = __ldg(a.in + e);
    __syncthreads();
    permute_lines<EPT, false>(sm, a.sched[0], a.logc, a.E[0], a.epw[0], a.w64[0], a.Ls);  // Step 1: rows
    permute_lines<EPT, true>(sm, a.sched[1], a.logr, a.E[1], a.epw[1], a.w64[1], a.Ls);   // Step 2: columns
    permute_lines<EPT, false>(sm, a.sched[2], a.logc, a.E[2], a.epw[2], a.w64[2], a.Ls);  // Step 3: rows
    for (int e = tid; e < n; e += T) a.out[e] = sm[(e >> a.logc) * a.Ls + (e & cmask)];
}

// ------------------------------------------------------------------ row pass

struct Io {
    int cross;
    int logw;                  // RUNS: log2 run width
    int logBP;                 // CROSS: log2 block of positions
    long long strideK;         // RUNS
    long long strideP;         // CROSS
    long long cta_stride;
};

struct RowArgs {
    const uint32_t* in;
    uint32_t* out;
    const uint32_t* sched;     // this pass's packed phase
    int logL, logh, Ls, E, epw, w64, dense;
    long long sched_words_per_cta;
    Io i, o;
    unsigned long long* trace;   // optional: 16 %globaltimer stamps per CTA (tracing)
    int in_segs;                 // >1: input line l of tile t = in_segs segments of seg_len
    long long seg_len, seg_stride;   //     at in + s*seg_stride + (t*h + l)*seg_len
};

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
// thread 0 of a CTA records stamp `slot` when tracing is enabled
__device__ __forceinline__ void stamp(unsigned long long* tr, int slot) {
    if (tr != nullptr && threadIdx.x == 0) tr[blockIdx.x * 16 + slot] = gtimer();
}

// Element (line l, position pos) of this CTA <-> global index (see plan.hpp IoMode).
// Vector v covers elements f = 4v .. 4v+3 of the CTA's flattened I/O order:
//   RUNS : f -> (K = f / (h*w), l = (f / w) % h, k = f % w), global base + K*strideK + f % (h*w)
//   CROSS: f -> (pos = f / h, l = f % h),             global base + (pos/BP)*strideP + f % (BP*h)
template <int EPT>
__device__ __forceinline__ void tile_load(const RowArgs& a, uint32_t* sm, long long cta) {
    const int T = blockDim.x, tid = threadIdx.x;
    const Io& m = a.i;
    const uint32_t* base = a.in + cta * m.cta_stride;
    constexpr int NV = EPT / 4;
    uint4 val[NV];
    if (a.in_segs > 1) {
        // sharded column phase: line l (global t*h + l) = in_segs segments of seg_len words
        // at in + s*seg_stride + (t*h + l)*seg_len (whole lines, m.w == L)
        const int logL = m.logw;
        const int logS = 31 - __clz((int)a.seg_len);
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int l = f >> logL, pos = f & ((1 << logL) - 1);
            const int s = pos >> logS, off = pos & ((1 << logS) - 1);
            val[it] = ld_nc_v4(a.in + s * a.seg_stride + (cta * (1 << a.logh) + l) * a.seg_len + off);
        }
    } else if (!m.cross) {
        const int loghw = a.logh + m.logw;
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int K = f >> loghw, rem = f & ((1 << loghw) - 1);
            val[it] = ld_nc_v4(base + (long long)K * m.strideK + rem);
        }
    }
    if (!m.cross) {
        const int loghw = a.logh + m.logw;
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int K = f >> loghw, rem = f & ((1 << loghw) - 1);
            const int l = rem >> m.logw, k = rem & ((1 << m.logw) - 1);
            *reinterpret_cast<uint4*>(sm + l * a.Ls + (K << m.logw) + k) = val[it];
        }
    } else {
        const int logBPh = m.logBP + a.logh;
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int pos = f >> a.logh;
            val[it] = ld_nc_v4(base + (long long)(pos >> m.logBP) * m.strideP +
                               (f & ((1 << logBPh) - 1)));
        }
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int pos = f >> a.logh, l = f & ((1 << a.logh) - 1);
            uint32_t* d = sm + l * a.Ls + pos;
            d[0] = val[it].x;
            d[a.Ls] = val[it].y;
            d[2 * a.Ls] = val[it].z;
            d[3 * a.Ls] = val[it].w;
        }
    }
}

template <int EPT>
__device__ __forceinline__ void tile_store(const RowArgs& a, const uint32_t* sm, long long cta) {
    const int T = blockDim.x, tid = threadIdx.x;
    const Io& m = a.o;
    uint32_t* base = a.out + cta * m.cta_stride;
    constexpr int NV = EPT / 4;
    if (!m.cross) {
        const int loghw = a.logh + m.logw;
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int K = f >> loghw, rem = f & ((1 << loghw) - 1);
            const int l = rem >> m.logw, k = rem & ((1 << m.logw) - 1);
            const uint4 v = *reinterpret_cast<const uint4*>(sm + l * a.Ls + (K << m.logw) + k);
            st_v4(base + (long long)K * m.strideK + rem, v);
        }
    } else {
        const int logBPh = m.logBP + a.logh;
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int pos = f >> a.logh, l = f & ((1 << a.logh) - 1);
            const uint32_t* s = sm + l * a.Ls + pos;
            uint4 v;
            v.x = s[0];
            v.y = s[a.Ls];
            v.z = s[2 * a.Ls];
            v.w = s[3 * a.Ls];
            st_v4(base + (long long)(pos >> m.logBP) * m.strideP + (f & ((1 << logBPh) - 1)), v);
        }
    }
}

// One row-wise permutation pass (Lemma 7): load h lines, permute each line in
// place with its bank-conflict-free schedule, store them in the next pass's layout.
template <int EPT>
__global__ void __launch_bounds__(512, (EPT <= 16) ? 2 : 1) row_pass_kernel(const RowArgs a) {
    extern __shared__ __align__(16) uint32_t sm[];
    const long long cta = blockIdx.x;
    const uint32_t* sched = a.sched + cta * a.sched_words_per_cta;
    // The schedule does not depend on the previous pass: pull it into L2 while
    // the previous kernel drains (32 words = one 128-byte line per thread step).
    for (long long w = (long long)threadIdx.x * 32; w < a.sched_words_per_cta;
         w += (long long)blockDim.x * 32)
        prefetch_l2(sched + w);
    stamp(a.trace, 0);
    pdl_wait();
    stamp(a.trace, 1);
    tile_load<EPT>(a, sm, cta);
    __syncthreads();
    stamp(a.trace, 2);
    pdl_launch_dependents();
    permute_lines<EPT, false>(sm, sched, a.logL, a.E, a.epw, a.w64, a.Ls, a.dense);
    stamp(a.trace, 3);
    tile_store<EPT>(a, sm, cta);
    stamp(a.trace, 14);
}

// ------------------------------------------------------------------ row pass, TMA pipeline

struct TmaArgs {
    RowArgs r;                 // geometry + output layout (r.o); r.i unused (input = lines)
    int ntiles, stages;
    int data_words;            // h * Ls
    int sched_words;           // h * (L/32) * E, a multiple of 4
    // half-line ring as a TLC pass (layout 5): each half of a permuted tile leaves as 3-D
    // tensor stores of its chunks into X1 / X2 (out_kind 1 / 2); 0 = 1-D bulk stores of rows
    int out_kind;
    int chunk, box_outer, box_words, boxes_per_half;
};

// Persistent, pipelined row-wise permutation pass (Lemma 7) for contiguous input
// lines. Each CTA walks tiles t = blockIdx.x + i*gridDim.x; a ring of `stages`
// shared-memory slots holds [h lines | the tile's packed schedule]. One thread
// arms the slot's mbarrier and issues TMA bulk copies (one per line, or one for
// the whole tile when unpadded, plus one for the schedule); while tile i is
// permuted and stored, tiles i+1 .. i+stages-1 are in flight. The schedule
// copy is issued before griddepcontrol.wait: it does not depend on the
// previous pass. Output: CROSS gather (column chunks of h elements, 128-bit
// stores) or, for row-major output, a TMA bulk store.
//
// SG (schedule from global): for long lines (L >= 16384, n >= 2^27) a slot holds
// the data only; the tile's schedule is pulled into L2 by a bulk prefetch when
// the slot is armed and read by the permuters straight from global memory
// (coalesced 64-bit loads), so two or three 64 KiB lines stay in flight per SM.
template <int EPT, bool OUT_CROSS, bool SG = false>
__global__ void __launch_bounds__(512, (EPT <= 16) ? 2 : 1) row_pass_tma_kernel(const TmaArgs a) {
    extern __shared__ __align__(128) uint32_t smem[];
    const int tid = threadIdx.x;
    const int L = 1 << a.r.logL, h = 1 << a.r.logh;
    const int stage_words = a.data_words + (SG ? 0 : a.sched_words);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + a.stages * stage_words);
    const int G = gridDim.x;
    const uint32_t line_bytes = (uint32_t)L * 4u;
    const bool dense = a.r.Ls == L;
    const uint32_t tile_bytes = (uint32_t)h * line_bytes + (SG ? 0u : (uint32_t)a.sched_words * 4u);

    auto issue_sched = [&](int s, long long t) {
        if constexpr (SG) {
            prefetch_l2_bulk(a.r.sched + t * a.sched_words, (uint32_t)a.sched_words * 4u);
        } else {
            bulk_g2s(smem + s * stage_words + a.data_words, a.r.sched + t * a.sched_words,
                     (uint32_t)a.sched_words * 4u, &bars[s]);
        }
    };
    auto issue_data = [&](int s, long long t) {
        uint32_t* dst = smem + s * stage_words;
        if (a.r.in_segs > 1) {
            const uint32_t sb = (uint32_t)a.r.seg_len * 4u;
            for (int l = 0; l < h; ++l)
                for (int g = 0; g < a.r.in_segs; ++g)
                    bulk_g2s(dst + l * a.r.Ls + g * a.r.seg_len,
                             a.r.in + g * a.r.seg_stride + (t * h + l) * a.r.seg_len, sb, &bars[s]);
            return;
        }
        const uint32_t* src = a.r.in + t * h * (long long)L;
        if (dense) {
            bulk_g2s(dst, src, (uint32_t)h * line_bytes, &bars[s]);
        } else {
            for (int l = 0; l < h; ++l) bulk_g2s(dst + l * a.r.Ls, src + (long long)l * L, line_bytes, &bars[s]);
        }
    };

    unsigned long long* tr = a.r.trace;
    stamp(tr, 0);
    if (tid == 0) {
        for (int s = 0; s < a.stages; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
        for (int s = 0; s < a.stages; ++s) {
            const long long t = blockIdx.x + (long long)s * G;
            if (t < a.ntiles) {
                mbar_arrive_expect_tx(&bars[s], tile_bytes);
                issue_sched(s, t);
            }
        }
    }
    pdl_wait();   // the previous pass's output is complete and visible from here on
    stamp(tr, 1);
    if (tid == 0) {
        for (int s = 0; s < a.stages; ++s) {
            const long long t = blockIdx.x + (long long)s * G;
            if (t < a.ntiles) issue_data(s, t);
        }
    }
    pdl_launch_dependents();
    for (int i = 0;; ++i) {
        const long long t = blockIdx.x + (long long)i * G;
        if (t >= a.ntiles) break;
        const int s = i % a.stages;
        mbar_wait(&bars[s], (uint32_t)(i / a.stages) & 1u);
        if (i < 4) stamp(tr, 2 + 3 * i);
        uint32_t* buf = smem + s * stage_words;
        if constexpr (SG)
            permute_lines<EPT, false, false>(buf, a.r.sched + t * a.sched_words, a.r.logL, a.r.E,
                                             a.r.epw, a.r.w64, a.r.Ls, a.r.dense);
        else
            permute_lines<EPT, false, true>(buf, buf + a.data_words, a.r.logL, a.r.E, a.r.epw,
                                            a.r.w64, a.r.Ls, a.r.dense);
        if (i < 4) stamp(tr, 3 + 3 * i);
        if constexpr (OUT_CROSS) {
            tile_store<EPT>(a.r, buf, t);
        } else {
            if (tid == 0) {
                fence_proxy_async();     // generic-proxy smem writes -> async-proxy reads
                uint32_t* dst = a.r.out + t * h * (long long)L;
                if (dense) {
                    bulk_s2g(dst, buf, (uint32_t)h * line_bytes);
                } else {
                    for (int l = 0; l < h; ++l) bulk_s2g(dst + (long long)l * L, buf + l * a.r.Ls, line_bytes);
                }
                bulk_commit();
            }
        }
        __syncthreads();                 // every thread is done with slot s
        if (i < 4) stamp(tr, 4 + 3 * i);
        if (tid == 0) {
            const long long tn = t + (long long)a.stages * G;
            if (tn < a.ntiles) {
                if constexpr (!OUT_CROSS) bulk_wait_read0();   // the bulk store has read slot s
                fence_proxy_async();
                mbar_arrive_expect_tx(&bars[s], tile_bytes);
                issue_sched(s, tn);
                issue_data(s, tn);
            }
        }
    }
    if constexpr (!OUT_CROSS) {
        if (tid == 0) bulk_wait0();
    }
    stamp(tr, 14);
}

// ------------------------------------------------------------------ row pass, half-line ring

// In-place permutation of ONE line whose two halves sit in shared-memory words
// [o0, o0 + L/2) and [o1, o1 + L/2) (any two slots of the half-line ring).
// Same warp-round structure and W64 schedule (read from global) as
// permute_lines; slots are 64 KiB apart, so position pos keeps bank pos mod 32
// and the rounds stay conflict-free.
template <int EPT, bool DENSE, bool KEEP, bool MERGE = false>
__device__ __forceinline__ void permute_split_line(uint32_t* sm, int o0, int o1, const uint32_t* __restrict__ sched,
                                                   int logL, int E, int epw, int w64) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, W = blockDim.x >> 5;
    const int lh = logL - 1;
    const int hmask = (1 << lh) - 1;
    const SchedDec dec(DENSE ? 1 : 0, E, epw, w64, lane);
    const uint32_t tmask = (1u << logL) - 1u;
    // one decode per format (compile time): W64 = one 64-bit load, dense = two 32-bit loads
    auto entry = [&](int q) -> uint32_t {
        if constexpr (DENSE) {
            const uint32_t* p = sched + q * E;
            const uint32_t lo = __ldg(p + dec.dwo), hi = __ldg(p + dec.dwo2);
            return (uint32_t)((((uint64_t)hi << 32) | lo) >> dec.dbo) & dec.mask;
        } else {
            const uint2 wd = __ldg(reinterpret_cast<const uint2*>(sched) + q * w64 + dec.wsel);
            return (uint32_t)((((uint64_t)wd.y << 32) | wd.x) >> dec.sh) & dec.mask;
        }
    };
    uint32_t v[EPT];
    if constexpr (MERGE && !DENSE && !KEEP) {
        // the first version of this kernel, verbatim: both hops load the same 64-bit words
        // through the same pointer arithmetic, which the compiler merges into one batch of
        // loads issued up front (measured 3.20 ms per pass at 2^30; rewrites with the
        // generic decoder compiled to heavier spilling, 4.7 ms)
        const uint2* sp = reinterpret_cast<const uint2*>(sched) + warp * w64 + dec.wsel;
        const int step = W * w64;
#pragma unroll
        for (int m = 0; m < EPT; ++m) {
            const uint2 wd = __ldg(sp + m * step);
            const uint64_t w = ((uint64_t)wd.y << 32) | wd.x;
            const uint32_t e = (uint32_t)(w >> dec.sh) & dec.mask;
            const int s = (int)((e >> logL) << 5) + lane;
            v[m] = sm[((s >> lh) ? o1 : o0) + (s & hmask)];
        }
        __syncthreads();
#pragma unroll
        for (int m = 0; m < EPT; ++m) {
            const uint2 wd = __ldg(sp + m * step);
            const uint64_t w = ((uint64_t)wd.y << 32) | wd.x;
            const int t = (int)(((uint32_t)(w >> dec.sh) & dec.mask) & tmask);
            sm[((t >> lh) ? o1 : o0) + (t & hmask)] = v[m];
        }
    } else if constexpr (KEEP) {
        // the schedule is read once: the destination word offsets (< 3 * 2^14 < 2^16)
        // wait in registers, two per register, across the barrier
        uint32_t ta[(EPT + 1) / 2];
#pragma unroll
        for (int m = 0; m < EPT; ++m) {
            const uint32_t e = entry(warp + W * m);
            const int s = (int)((e >> logL) << 5) + lane;
            v[m] = sm[((s >> lh) ? o1 : o0) + (s & hmask)];
            const int t = (int)(e & tmask);
            const uint32_t ad = (uint32_t)(((t >> lh) ? o1 : o0) + (t & hmask));
            if (m & 1) ta[m >> 1] |= ad << 16;
            else ta[m >> 1] = ad;
        }
        __syncthreads();
#pragma unroll
        for (int m = 0; m < EPT; ++m) sm[(ta[m >> 1] >> ((m & 1) * 16)) & 0xFFFFu] = v[m];
    } else {
#pragma unroll
        for (int m = 0; m < EPT; ++m) {
            const uint32_t e = entry(warp + W * m);
            const int s = (int)((e >> logL) << 5) + lane;
            v[m] = sm[((s >> lh) ? o1 : o0) + (s & hmask)];
        }
        __syncthreads();
        // MERGE: the write hop names the same addresses, so the compiler issues each
        // schedule load once, all up front (measured fastest at L = 32768 with W64
        // entries, although it parks part of them in local memory); otherwise the
        // loads are re-issued after the barrier (warp index laundered through a shuffle)
        const int warp2 = MERGE ? warp : __shfl_sync(kFull, warp, 0);
#pragma unroll
        for (int m = 0; m < EPT; ++m) {
            const int t = (int)(entry(warp2 + W * m) & tmask);
            sm[((t >> lh) ? o1 : o0) + (t & hmask)] = v[m];
        }
    }
    __syncthreads();
}

// Row-wise pass (Lemma 7) for lines of L = 32768 words (n = 2^29, 2^30), where one
// line + any second buffer exceed shared memory: a ring of THREE half-line slots
// (3 x 64 KiB). Line i occupies slots (2i mod 3, 2i+1 mod 3); while line i is
// permuted, the first half of line i+1 is already loading into the third slot;
// once the TMA store of line i's first half has read its slot, the second half
// of line i+1 loads there, and once the second half's store has read its slot,
// the first half of line i+2 loads there. So loads overlap the permute and the
// stores instead of alternating with them (1.5 lines resident per SM).
// Half-load j = 2i + q uses slot j mod 3 and is that slot's (j div 3)-th fill:
// the mbarrier parity every thread waits on is (j div 3) & 1. Schedule: W64,
// read from global, L2-prefetched one line ahead. Row-major output only.
template <int EPT, bool DENSE, bool KEEP>
__global__ void __launch_bounds__((EPT >= 64) ? 512 : 1024, 1) row_pass_split_kernel(const TmaArgs a) {
    // !DENSE && !KEEP: W64 entries, loads merged across the two hops (the default)
    constexpr bool MERGE = !DENSE && !KEEP;
    extern __shared__ __align__(128) uint32_t smem[];
    const int tid = threadIdx.x;
    const int L = 1 << a.r.logL, HALF = L >> 1, lh = a.r.logL - 1;
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + 3 * HALF);
    const int G = gridDim.x;
    const uint32_t half_bytes = (uint32_t)HALF * 4u;
    const long long my_lines = a.ntiles > (int)blockIdx.x ? (a.ntiles - 1 - (int)blockIdx.x) / G + 1 : 0;

    // half-load j of this CTA: line j >> 1, half j & 1, slot j % 3
    auto issue_half = [&](long long j) {
        const long long i = j >> 1;
        if (i >= my_lines) return;
        const int q = (int)(j & 1), slot = (int)(j % 3);
        const long long t = blockIdx.x + i * G;
        uint32_t* dst = smem + slot * HALF;
        mbar_arrive_expect_tx(&bars[slot], half_bytes);
        if (q == 0) prefetch_l2_bulk(a.r.sched + t * a.sched_words, (uint32_t)a.sched_words * 4u);
        if (a.r.in_segs > 1) {
            const uint32_t sb = (uint32_t)a.r.seg_len * 4u;
            for (int g = 0; g < a.r.in_segs; ++g) {
                const long long off = (long long)g * a.r.seg_len;
                if ((off >> lh) != q) continue;
                bulk_g2s(dst + (off & (HALF - 1)), a.r.in + g * a.r.seg_stride + t * a.r.seg_len, sb, &bars[slot]);
            }
        } else {
            bulk_g2s(dst, a.r.in + t * (long long)L + (long long)q * HALF, half_bytes, &bars[slot]);
            if (q == 0) prefetch_l2_bulk(a.r.in + t * (long long)L + HALF, half_bytes);
        }
    };

    unsigned long long* tr = a.r.trace;
    stamp(tr, 0);
    if (tid == 0) {
        for (int s = 0; s < 3; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
        if (my_lines > 0) prefetch_l2_bulk(a.r.sched + (long long)blockIdx.x * a.sched_words,
                                           (uint32_t)a.sched_words * 4u);
    }
    __syncthreads();
    pdl_wait();
    stamp(tr, 1);
    if (tid == 0) {
        issue_half(0);
        issue_half(1);
        issue_half(2);
    }
    pdl_launch_dependents();
    for (long long i = 0; i < my_lines; ++i) {
        const long long t = blockIdx.x + i * G;
        const long long j0 = 2 * i, j1 = 2 * i + 1;
        const int s0 = (int)(j0 % 3), s1 = (int)(j1 % 3);
        mbar_wait(&bars[s0], (uint32_t)(j0 / 3) & 1u);
        mbar_wait(&bars[s1], (uint32_t)(j1 / 3) & 1u);
        if (i < 4) stamp(tr, 2 + 3 * i);
        permute_split_line<EPT, DENSE, KEEP, MERGE>(smem, s0 * HALF, s1 * HALF, a.r.sched + t * a.sched_words,
                                                    a.r.logL, a.r.E, a.r.epw, a.r.w64);
        if (i < 4) stamp(tr, 3 + 3 * i);
        if (tid == 0) {
            fence_proxy_async();     // generic-proxy smem writes -> async-proxy reads
            uint32_t* dst = a.r.out + t * (long long)L;
            bulk_s2g(dst, smem + s0 * HALF, half_bytes);
            bulk_commit();
            bulk_s2g(dst + HALF, smem + s1 * HALF, half_bytes);
            bulk_commit();
            bulk_wait_read1();       // first half read out of slot s0
            fence_proxy_async();
            issue_half(2 * i + 3);   // second half of line i+1 -> slot s0
            bulk_wait_read0();       // second half read out of slot s1
            fence_proxy_async();
            issue_half(2 * i + 4);   // first half of line i+2 -> slot s1
        }
        if (i < 4) stamp(tr, 4 + 3 * i);
    }
    if (tid == 0) bulk_wait0();
    stamp(tr, 14);
}

// ------------------------------------------------------------------ named barriers, mbarrier arrive, trace stamps

__device__ __forceinline__ void named_bar(int id, int count) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void stamp_if(unsigned long long* tr, bool who, int slot) {
    if (tr != nullptr && who) tr[blockIdx.x * 16 + slot] = gtimer();
}

// ------------------------------------------------------------------ half-line ring, staged schedule

constexpr int kStgWorkers = 512;                 // 16 warps
constexpr int kStgChunkWords = 2048;             // W64: 8 KiB schedule chunks (64 rounds of 16 words)
constexpr int kStgDenseWords = 64 * 25;          // dense: 64 rounds of E <= 25 words (6.25 KiB)

// Half-line ring (row_pass_split_kernel) with the schedule STREAMED THROUGH SHARED MEMORY:
// the 35 KiB left beside the three 64 KiB half-line slots hold a ring of schedule chunks
// (W64: four of 8 KiB; dense: five of 64*E words) filled with TMA bulk copies. One chunk =
// 64 warp-rounds = 4 rounds of each of the 16 warps; the ring runs ahead into the next line
// while the current one is written back. Thread 0 refills a buffer once all 512 threads have
// arrived on its `empty` mbarrier (16 warps = 4 per SM quadrant keep 128 registers per
// thread). Each entry is read once from shared memory and the decoded destination offsets
// stay in registers across the barrier. The permute is bound by the chunk latency (per-CTA
// traces, profiles/r01_trace_ring_s8.log), hence the dense format's smaller, deeper ring.
template <int EPT, bool DENSE>
__global__ void __launch_bounds__(kStgWorkers, 1)
    row_pass_split_stg_kernel(const __grid_constant__ CUtensorMap tmap, const TmaArgs a) {
    extern __shared__ __align__(128) uint32_t smem[];
    constexpr int NB = DENSE ? 5 : 4;            // chunk ring depth
    constexpr int CWS = DENSE ? kStgDenseWords : kStgChunkWords;   // buffer stride (words)
    const int tid = threadIdx.x;
    // geometry from EPT (one line of L = 512 * EPT words per CTA; entries of the full
    // per-line format, E = 2 log2 L - 5 bits; launch_row_pass checks the plan agrees):
    // compile-time shifts and masks in the decode and the half-slot addressing
    constexpr int LOGL = cilog2(kStgWorkers * EPT);
    constexpr int L = 1 << LOGL, HALF = L >> 1, lh = LOGL - 1, hmask = HALF - 1;
    constexpr int E = 2 * LOGL - 5;
    constexpr int CW = DENSE ? 64 * E : kStgChunkWords;             // words per chunk
    uint32_t* cbuf = smem + 3 * HALF;
    uint64_t* bars = reinterpret_cast<uint64_t*>(cbuf + NB * CWS);
    uint64_t* full = bars + 3;                   // chunk landed
    // chunk buffer b's consumption count (warps; monotone): the warp whose arrival completes
    // a multiple of 16 refills the buffer itself -- no thread blocks waiting for the others
    uint32_t* consumed = reinterpret_cast<uint32_t*>(bars + 3 + NB);
    const int G = gridDim.x;
    const uint32_t half_bytes = (uint32_t)HALF * 4u;
    const long long my_lines = a.ntiles > (int)blockIdx.x ? (a.ntiles - 1 - (int)blockIdx.x) / G + 1 : 0;
    constexpr int kW = kStgWorkers / 32;                   // warps
    const int w64 = a.r.w64;
    constexpr int chunks_per_line = EPT / 4;     // (L/32 rounds) / 64 rounds per chunk

    // half q of line i -> slot j % 3. With the first half, the line's second half is pulled
    // into L2: its TMA load can only be issued once the previous line's first half has been
    // stored out of its slot, and then it hits L2 instead of HBM. Sharded column phases
    // (in_segs > 1): a line is in_segs segments of seg_len <= L/2 words, one per sender.
    auto issue_half = [&](long long j) {
        const long long i = j >> 1;
        if (i >= my_lines) return;
        const int q = (int)(j & 1), slot = (int)(j % 3);
        const long long t = blockIdx.x + i * G;
        uint32_t* dst = smem + slot * HALF;
        mbar_arrive_expect_tx(&bars[slot], half_bytes);
        if (q == 0) prefetch_l2_bulk(a.r.sched + t * a.sched_words, (uint32_t)a.sched_words * 4u);
        if (a.r.in_segs > 1) {
            const uint32_t sb = (uint32_t)a.r.seg_len * 4u;
            for (int g = 0; g < a.r.in_segs; ++g) {
                const long long off = (long long)g * a.r.seg_len;
                const uint32_t* src = a.r.in + g * a.r.seg_stride + t * a.r.seg_len;
                if ((off >> lh) == q) bulk_g2s(dst + (off & (HALF - 1)), src, sb, &bars[slot]);
                else if (q == 0) prefetch_l2_bulk(src, sb);
            }
        } else {
            const uint32_t* src = a.r.in + t * (long long)L;
            bulk_g2s(dst, src + (long long)q * HALF, half_bytes, &bars[slot]);
            if (q == 0) prefetch_l2_bulk(src + HALF, half_bytes);
        }
    };

    unsigned long long* tr = a.r.trace;
    stamp(tr, 0);
    if (tid == 0) {
        for (int s = 0; s < 3; ++s) mbar_init(&bars[s], 1);
        for (int b = 0; b < NB; ++b) {
            mbar_init(&full[b], 1);
            consumed[b] = 0;
        }
        fence_mbar_init();
        if (my_lines > 0) prefetch_l2_bulk(a.r.sched + (long long)blockIdx.x * a.sched_words,
                                           (uint32_t)a.sched_words * 4u);
    }
    __syncthreads();
    const long long total_chunks = my_lines * chunks_per_line;
    auto issue_chunk = [&](long long g, int b) {      // b = g % NB
        const long long i = g / chunks_per_line, c = g - i * chunks_per_line;
        const long long t = blockIdx.x + i * G;
        mbar_arrive_expect_tx(&full[b], (uint32_t)CW * 4u);
        bulk_g2s(cbuf + b * CWS, a.r.sched + t * a.sched_words + c * CW, (uint32_t)CW * 4u, &full[b]);
    };
    if (tid == 0)
        for (long long g = 0; g < NB && g < total_chunks; ++g) issue_chunk(g, (int)g);
    pdl_wait();
    stamp(tr, 1);
    if (tid == 0) {
        issue_half(0);
        issue_half(1);
        issue_half(2);
    }
    pdl_launch_dependents();
    const int lane = tid & 31, warp = tid >> 5;
    const SchedDec dec(DENSE ? 1 : 0, E, a.r.epw, w64, lane);
    constexpr uint32_t tmask = (1u << LOGL) - 1u;
    constexpr uint32_t EMASK = (1u << E) - 1u;
    constexpr int logL = LOGL;
    constexpr int MPC = 4;               // m-steps per chunk: 64 rounds = 4 x 16 warps
    constexpr int CPL = EPT / MPC;       // chunks per line
    // dense entries: the lane's entry of round q of a chunk starts at bit lane*E of the
    // round's E words: words dwo, dwo2 (= dwo or dwo + 1) at warp*E (+ 16*E per m-step)
    const int lane_w0 = warp * E + dec.dwo, lane_w1 = warp * E + dec.dwo2;
    const uint32_t lane_sh = (uint32_t)dec.dbo;
    long long g = 0;                     // this CTA's chunk sequence number
    int cb_i = 0;                        // g % NB
    uint32_t cb_ph = 0;                  // (g / NB) & 1
    for (long long i = 0; i < my_lines; ++i) {
        const long long t = blockIdx.x + i * G;
        const long long j0 = 2 * i, j1 = 2 * i + 1;
        const int s0 = (int)(j0 % 3), s1 = (int)(j1 % 3);
        const int o0 = s0 * HALF, o1 = s1 * HALF;
        mbar_wait(&bars[s0], (uint32_t)(j0 / 3) & 1u);
        mbar_wait(&bars[s1], (uint32_t)(j1 / 3) & 1u);
        if (i < 4) stamp(tr, 2 + 3 * (int)i);
        uint32_t v[EPT];
        uint32_t ta[EPT / 2];
#pragma unroll
        for (int c = 0; c < CPL; ++c, ++g) {
            const int b = cb_i;
            mbar_wait(&full[b], cb_ph);
            const uint32_t* cb = cbuf + b * CWS;
#pragma unroll
            for (int mm = 0; mm < MPC; ++mm) {
                const int m = c * MPC + mm;
                uint32_t e;
                if constexpr (DENSE) {
                    const uint32_t lo = cb[lane_w0 + mm * kW * E], hi = cb[lane_w1 + mm * kW * E];
                    e = __funnelshift_r(lo, hi, lane_sh) & EMASK;
                } else {
                    e = dec.get<true>(cb, warp + kW * mm);
                }
                const int s = (int)((e >> logL) << 5) + lane;
                v[m] = smem[((s >> lh) ? o1 : o0) + (s & hmask)];
                const int tt = (int)(e & tmask);
                const uint32_t ad = (uint32_t)(((tt >> lh) ? o1 : o0) + (tt & hmask));
                if (m & 1) ta[m >> 1] |= ad << 16;
                else ta[m >> 1] = ad;
            }
            if (c == 0 && i > 0 && tid == 0) {
                // line i-1's second half (slot s1 of line i-1 = the slot of line i+1's first
                // half) was handed to its TMA store at the end of line i-1; by now it has been
                // read out, so this wait no longer holds warp 0 back at the line boundary
                bulk_wait_read0();
                fence_proxy_async();
                issue_half(2 * i + 2);
            }
            __syncwarp();                     // the warp's reads of chunk g precede lane 0's release
            if (lane == 0 && g + NB < total_chunks) {
                uint32_t old;
                asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], 1;"
                             : "=r"(old) : "r"(smem_u32(&consumed[b])) : "memory");
                if ((old + 1) % kW == 0) {       // the last of the 16 warps to consume chunk g
                    fence_proxy_async();         // all warps' generic reads -> the TMA refill
                    issue_chunk(g + NB, b);
                }
            }
            if (++cb_i == NB) { cb_i = 0; cb_ph ^= 1u; }
        }
        __syncthreads();
#pragma unroll
        for (int m = 0; m < EPT; ++m) smem[(ta[m >> 1] >> ((m & 1) * 16)) & 0xFFFFu] = v[m];
        __syncthreads();
        if (i < 4) stamp(tr, 3 + 3 * (int)i);
        if (tid == 0) {
            fence_proxy_async();
            if (a.out_kind == 0) {
                uint32_t* dst = a.r.out + t * (long long)L;
                bulk_s2g(dst, smem + o0, half_bytes);
                bulk_commit();
                bulk_s2g(dst + HALF, smem + o1, half_bytes);
                bulk_commit();
            } else {
                // the tile's output order is its chunks (one per K- / I'-block) back to back;
                // half q holds blocks [q * nbh, (q + 1) * nbh), nbh = boxes_per_half * box_outer
                for (int q = 0; q < 2; ++q) {
                    const uint32_t* src = smem + (q ? o1 : o0);
                    for (int bx = 0; bx < a.boxes_per_half; ++bx)
                        tma_store_3d(&tmap, src + bx * a.box_words, 0, (int)t * a.chunk,
                                     (q * a.boxes_per_half + bx) * a.box_outer);
                    bulk_commit();
                }
            }
            bulk_wait_read1();
            fence_proxy_async();
            issue_half(2 * i + 3);           // second half of line i+1 -> slot s0
            // the first half of line i+2 (-> slot s1, once the second store has read it) is
            // issued by thread 0 after its first schedule chunk of line i+1
        }
        if (i < 4) stamp(tr, 4 + 3 * (int)i);
    }
    if (tid == 0) bulk_wait0();
    stamp(tr, 14);
}

// ------------------------------------------------------------------ fused 3-pass persistent kernel

__device__ __forceinline__ void fence_proxy_async_global() {
    asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_gpu(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_release_gpu_add(unsigned long long* p, unsigned long long v) {
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_relaxed_gpu_add(unsigned long long* p, unsigned long long v) {
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// ------------------------------------------------------------------ TLC row pass (tile-level colouring)



struct TlcArgs {
    const uint32_t* in;
    uint32_t* out;             // row-major output (OUT == 0)
    const uint32_t* sched;
    int ntiles, na, nb;        // A slots (loads in flight), B slots (stores in flight)
    long long tile_words;      // schedule words per tile
    int chunk;                 // box rows per tile chunk (chunk words / box row words)
    int nbox, box_outer, box_words;
    unsigned long long* trace;
    int prefetch_in;           // stream the whole input into L2 up front (HBM-resident input)
    int segs;                  // > 1: tile t = segs segments of seg_len words (sharded, plan.hpp)
    long long seg_len, seg_stride;
    TlcDecode dec;             // entry -> destination (plan.hpp)
};

// Shared-memory word offsets of the TLC rings: A slots, then B slots, then mbarriers.
struct TlcRing {
    uint32_t* A;
    uint32_t* B;
    uint64_t* afull;           // TMA bytes of A slot landed        (producer arms, TMA completes)
    uint64_t* aempty;          // A slot read by all permuters      (kTlcPerm arrivals)
    uint64_t* bfull;           // B slot written by all permuters   (kTlcPerm arrivals)
    uint64_t* bempty;          // B slot read by its TMA store      (storer arrives)
    __device__ TlcRing(uint32_t* smem, int HL, int na, int nb) {
        A = smem;
        B = smem + (size_t)na * HL;
        afull = reinterpret_cast<uint64_t*>(B + (size_t)nb * HL);
        aempty = afull + na;
        bfull = aempty + na;
        bempty = bfull + nb;
    }
    __device__ void init(int na, int nb) {
        for (int s = 0; s < na; ++s) {
            mbar_init(&afull[s], 1);
            mbar_init(&aempty[s], kTlcPerm);
        }
        for (int s = 0; s < nb; ++s) {
            mbar_init(&bfull[s], kTlcPerm);
            mbar_init(&bempty[s], 1);
        }
        fence_mbar_init();
    }
};

// TMA store of a permuted tile t from B slot `B` (see TlcArgs / make_tlc_maps):
// kind 0 = one 1-D bulk store of a row-major tile, kind 1/2 = 3-D tensor stores
// whose box rows are the tile's contiguous chunks (h1*h2 or h3*h2 words, split
// into `chunk` rows of at most 256 words).
__device__ __forceinline__ void tlc_store(int kind, const CUtensorMap* map, uint32_t* out, const uint32_t* B,
                                          long long t, int HL, int chunk, int nbox, int box_outer,
                                          int box_words) {
    if (kind == 0) {
        bulk_s2g(out + t * HL, B, (uint32_t)HL * 4u);
    } else {
        for (int b = 0; b < nbox; ++b)
            tma_store_3d(map, B + b * box_words, 0, (int)(t * chunk), b * box_outer);
    }
    bulk_commit();
}

// Permute one tile: A (TMA-loaded, the pass's input order) -> B (the pass's
// output order). Warp-round m of permuter warp pw: lane x reads A[32*sigma + x]
// (bank x) and writes B[dst] (32 distinct banks per round, by construction of
// the tile-level colouring). Entries are decoded from the lane's bitstream `wc`.
// Entry decode variants (plan.hpp TlcDecode), chosen at compile time:
//   TLC_FULL: entry = (sigma << log2 HL) | dst
//   TLC_X1 / TLC_X2 / TLC_ROWS: compact entries of pass 1 / 2 / 3, entry = (sigma << lt) | t,
//   dst rebuilt with the line index taken from sigma (X1) or from the lane (X2, ROWS; a
//   per-lane constant `lc`, so those decodes cost no more than the full format)
enum { TLC_FULL = 0, TLC_X1 = 1, TLC_X2 = 2, TLC_ROWS = 3 };

__device__ __forceinline__ uint32_t tlc_lane_const(int kind, const TlcDecode& dc, int lane) {
    if (kind == TLC_X2) return (uint32_t)lane & dc.m2;
    if (kind == TLC_ROWS) return (((uint32_t)lane >> dc.s4) & dc.m2) << dc.s3;
    return 0u;
}

template <int EPT, int E, int KIND>
__device__ __forceinline__ void tlc_permute(const uint32_t* __restrict__ A, uint32_t* __restrict__ B,
                                            const uint32_t* wc, const TlcDecode& dc, uint32_t lc,
                                            uint64_t* aempty, uint64_t* bempty_wait, uint32_t bparity,
                                            int lane) {
    constexpr int HL = kTlcPerm * EPT;
    constexpr int LOGHL = cilog2(HL);
    constexpr uint32_t EMASK = (1u << E) - 1u;
    const int lt = KIND == TLC_FULL ? LOGHL : dc.lt;
    const uint32_t tmask = KIND == TLC_FULL ? (uint32_t)(HL - 1) : (1u << dc.lt) - 1u;
    const int sh_line = dc.lt + dc.s4 - 5;    // TLC_X1: line index = e >> sh_line
    // Beyond 16 elements per thread the tile is moved in groups of 16 (read 16, write 16),
    // so that two tiles' schedule words + one group's values fit in 96 registers.
    constexpr int GRP = EPT <= 16 ? EPT : 16;
    uint32_t v[GRP];
    uint32_t d[GRP];
#pragma unroll
    for (int g0 = 0; g0 < EPT; g0 += GRP) {
#pragma unroll
        for (int j = 0; j < GRP; ++j) {
            const int m = g0 + j;
            const int bit = m * E, w = bit >> 5, off = bit & 31;
            uint32_t e;
            if (off + E <= 32) e = (wc[w] >> off) & EMASK;
            else e = __funnelshift_r(wc[w], wc[w + 1], off) & EMASK;
            const uint32_t t = e & tmask;
            v[j] = A[((e >> lt) << 5) | (uint32_t)lane];
            if constexpr (KIND == TLC_FULL) d[j] = t;
            else if constexpr (KIND == TLC_X2) d[j] = (t << dc.s2) | lc;
            else if constexpr (KIND == TLC_ROWS) d[j] = t | lc;
            else d[j] = ((t >> dc.s1) << dc.s2) | ((e >> sh_line) << dc.s3) | (t & dc.m1);
        }
        if (g0 + GRP == EPT) mbar_arrive(aempty);     // A slot may be refilled
        if (g0 == 0 && bempty_wait) mbar_wait(bempty_wait, bparity);
#pragma unroll
        for (int j = 0; j < GRP; ++j) B[d[j]] = v[j];
    }
    fence_proxy_async();                      // generic-proxy writes -> the TMA store's reads
}

// One row-wise permutation pass (Lemma 7) with the tile-level bank colouring
// (plan.hpp TlcPass). A tile of h lines is TMA-loaded into an A slot in its
// global order; 512 permuter threads move every element A[src] -> B[dst] in
// warp-rounds that touch 32 distinct banks of A and 32 distinct banks of B;
// B is already in the global order of the output, so the transposes of the
// column-wise step (Lemma 8) cost nothing extra: B leaves by TMA (1-D bulk
// store for row-major output, 2-D tensor stores of 64-byte chunks for the
// intermediates). Roles: warp 0 lane 0 = TMA producer, warp 1 lane 0 = TMA
// storer, warps 2..17 = permuters. Separate rings: `na` A slots (a CTA's whole
// share of tiles is requested up front when it fits) and `nb` B slots.
template <int EPT, int OUT, int E>
__global__ void __launch_bounds__(64 + kTlcPerm, 1)
    row_pass_tlc_kernel(const __grid_constant__ CUtensorMap tmap, const TlcArgs a) {
    constexpr int HL = kTlcPerm * EPT;
    constexpr int NWORDS = (EPT * E + 31) / 32;
    extern __shared__ __align__(128) uint32_t smem[];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NA = a.na, NB = a.nb;
    const int G = gridDim.x;
    TlcRing R(smem, HL, NA, NB);
    unsigned long long* tr = a.trace;
    stamp(tr, 0);
    if (tr != nullptr && tid == 0) {          // trace slot 15: the SM this CTA runs on
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        tr[blockIdx.x * 16 + 15] = smid;
    }
    if (tid == 0) R.init(NA, NB);
    __syncthreads();

    if (warp == 0) {
        if (lane == 0) {
            // ---------------- producer
            // Schedules do not depend on the previous pass. L2-resident input (passes 2, 3):
            // every schedule chunk of this CTA is requested into L2 before griddepcontrol.wait,
            // using HBM while the previous pass drains. HBM-resident input (pass 1): data and
            // schedule compete for HBM, so only the first two tiles' schedules go ahead and
            // the rest are interleaved behind the data loads (first tile lands earlier).
            const int sched_ahead = a.prefetch_in ? 2 : (1 << 30);
            auto prefetch_sched = [&](int i) {
                const long long t = blockIdx.x + (long long)i * G;
                if (t < a.ntiles) prefetch_l2_bulk(a.sched + t * a.tile_words, (uint32_t)(a.tile_words * 4));
            };
            for (int i = 0; i < sched_ahead; ++i) {
                if (blockIdx.x + (long long)i * G >= a.ntiles) break;
                prefetch_sched(i);
            }
            pdl_wait();
            stamp(tr, 1);
            for (int i = 0;; ++i) {
                const long long t = blockIdx.x + (long long)i * G;
                if (t >= a.ntiles) break;
                const int s = i % NA;
                if (i >= NA) mbar_wait(&R.aempty[s], (uint32_t)(i / NA - 1) & 1u);
                fence_proxy_async();           // permuters' generic reads of the slot -> TMA write
                mbar_arrive_expect_tx(&R.afull[s], (uint32_t)HL * 4u);
                if (a.segs > 1) {              // one segment per sender, in sender order
                    for (int g = 0; g < a.segs; ++g)
                        bulk_g2s(R.A + (size_t)s * HL + g * a.seg_len, a.in + g * a.seg_stride + t * a.seg_len,
                                 (uint32_t)a.seg_len * 4u, &R.afull[s]);
                } else {
                    bulk_g2s(R.A + (size_t)s * HL, a.in + t * HL, (uint32_t)HL * 4u, &R.afull[s]);
                }
                if (i == 0) pdl_launch_dependents();
                if (a.prefetch_in) {
                    prefetch_sched(i + sched_ahead);
                    if (i + 1 == NA)           // input tiles beyond the ring: into L2 now
                        for (int j = NA;; ++j) {
                            const long long tj = blockIdx.x + (long long)j * G;
                            if (tj >= a.ntiles) break;
                            prefetch_l2_bulk(a.in + tj * HL, (uint32_t)HL * 4u);
                        }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ---------------- storer: at most one store un-read while the next is issued
            pdl_wait();
            int prev = -1;
            for (int i = 0;; ++i) {
                const long long t = blockIdx.x + (long long)i * G;
                if (t >= a.ntiles) break;
                const int s = i % NB;
                mbar_wait(&R.bfull[s], (uint32_t)(i / NB) & 1u);
                tlc_store(OUT, &tmap, a.out, R.B + (size_t)s * HL, t, HL, a.chunk, a.nbox, a.box_outer,
                          a.box_words);
                if (NB == 1) {
                    bulk_wait_read0();
                    mbar_arrive(&R.bempty[s]);
                } else {
                    if (prev >= 0) {
                        bulk_wait_read1();
                        mbar_arrive(&R.bempty[prev]);
                    }
                    prev = s;
                }
                if (i < 4) stamp_if(tr, true, 4 + 3 * i);
            }
            stamp_if(tr, true, 12);           // last store issued
            bulk_wait0();
            stamp_if(tr, true, 13);           // every store of this CTA complete
        }
    } else {
        // ---------------- permuters
        constexpr int KIND = (E == 2 * cilog2(HL) - 5) ? TLC_FULL
                             : (OUT == 1 ? TLC_X1 : (OUT == 2 ? TLC_X2 : TLC_ROWS));
        const uint32_t lc = tlc_lane_const(KIND, a.dec, lane);
        const bool lead = tid == 64;
        const uint32_t* sp = a.sched + (warp - 2) * NWORDS * 32 + lane;
        // schedule words live in registers, loaded AHEAD tiles ahead (L2 latency under the
        // load of a pass is about one tile period); each is read once, so it leaves L2 first
        // (the intermediates X1 / X2 are what the next pass reads)
        const uint64_t pol_first = policy_evict_first();
        constexpr int AHEAD = NWORDS <= 12 ? 2 : 1;
        constexpr int NBUF = AHEAD + 1;
        // The buffers rotate by unrolling the tile loop NBUF times (compile-time buffer
        // indices): copying a buffer that has loads in flight (wq[k] = wq[k + 1]) would
        // stall every tile on the previous tile's schedule loads (an L2 round trip).
        uint32_t wq[NBUF][NWORDS];
#pragma unroll
        for (int k = 0; k < AHEAD; ++k) {
            const long long tk = blockIdx.x + (long long)k * G;
            if (tk < a.ntiles) {
#pragma unroll
                for (int w = 0; w < NWORDS; ++w) wq[k][w] = ld_nc_hint(sp + tk * a.tile_words + w * 32, pol_first);
            }
        }
        int s = 0, sb = 0;                    // A / B slots of tile i
        uint32_t pa = 0u, pb = 1u;            // afull parity of slot s, bempty parity of slot sb
        for (int i0 = 0;; i0 += NBUF) {
            bool done = false;
#pragma unroll
            for (int u = 0; u < NBUF; ++u) {
                const int i = i0 + u;
                const long long t = blockIdx.x + (long long)i * G;
                if (t >= a.ntiles) { done = true; break; }
                const long long tn = t + (long long)AHEAD * G;
                if (tn < a.ntiles) {
#pragma unroll
                    for (int w = 0; w < NWORDS; ++w)
                        wq[(u + AHEAD) % NBUF][w] = ld_nc_hint(sp + tn * a.tile_words + w * 32, pol_first);
                }
                mbar_wait(&R.afull[s], pa);
                if (i < 4) stamp_if(tr, lead, 2 + 3 * i);
                tlc_permute<EPT, E, KIND>(R.A + (size_t)s * HL, R.B + (size_t)sb * HL, wq[u], a.dec, lc,
                                          &R.aempty[s], i >= NB ? &R.bempty[sb] : nullptr, pb, lane);
                mbar_arrive(&R.bfull[sb]);
                if (++s == NA) { s = 0; pa ^= 1u; }
                if (++sb == NB) { sb = 0; pb ^= 1u; }
            }
            if (done) break;
        }
        stamp_if(tr, lead, 3);
    }
    stamp(tr, 14);
}

// ------------------------------------------------------------------ TLC, all three passes in one launch

struct TlcPassCfg {
    const uint32_t* in;
    uint32_t* out;             // row-major output (kind 0)
    const uint32_t* sched;
    int ntiles;
    int kind;                  // 0: rows (1-D bulk store), 1: X1, 2: X2 (3-D tensor stores)
    int chunk, nbox, box_outer, box_words;
    TlcDecode dec;
};

struct TlcFusedArgs {
    TlcPassCfg p[3];
    long long tile_words;
    int na, nb;
    unsigned long long* sync;  // [0], [1]: barrier arrivals after pass 0 / 1; [2]: exits
    unsigned long long* trace;
};

// Thm 9 in ONE persistent launch with the TLC passes (square views: the three
// passes share the tile size HL). Same roles and rings as row_pass_tlc_kernel,
// continued across passes (global tile sequence j). The storer publishes a
// CTA's pass-k output once its bulk stores have COMPLETED (wait_group 0, then a
// release at gpu scope on sync[k]); the producer TMA-loads pass k+1 data only
// after sync[k] reaches the grid size (schedule prefetches go ahead of the
// barrier). One co-resident CTA per SM; the last CTA out resets the counters,
// so the launch is replayable (CUDA graphs).
template <int EPT, int E>
__global__ void __launch_bounds__(64 + kTlcPerm, 1)
    fused_tlc_kernel(const __grid_constant__ CUtensorMap map_x1,
                     const __grid_constant__ CUtensorMap map_x2, const TlcFusedArgs a) {
    constexpr int HL = kTlcPerm * EPT;
    constexpr int NWORDS = (EPT * E + 31) / 32;
    extern __shared__ __align__(128) uint32_t smem[];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NA = a.na, NB = a.nb;
    const int G = gridDim.x;
    TlcRing R(smem, HL, NA, NB);
    uint64_t* pdone = R.bempty + NB;   // [k]: this CTA's pass-k stores are complete and published
    unsigned long long* tr = a.trace;
    stamp(tr, 0);
    if (tid == 0) {
        mbar_init(&pdone[0], 1);
        mbar_init(&pdone[1], 1);
        R.init(NA, NB);
    }
    __syncthreads();
    auto my_tiles = [&](int k) -> int {
        const int nt = a.p[k].ntiles - (int)blockIdx.x;
        return nt > 0 ? (nt + G - 1) / G : 0;
    };

    if (warp == 0) {
        if (lane == 0) {
            // ---------------- producer
            // Schedules are independent of the data. Pass 0 (HBM input): the first two tiles'
            // schedules go ahead, the rest interleave behind the data loads, input tiles beyond
            // the ring are streamed into L2. Pass k + 1's schedules are requested once this
            // CTA's last pass-k tile has landed (HBM free of this CTA's pass-k traffic), ahead of
            // the grid barrier.
            auto prefetch_one = [&](int k, int i) {
                if (i < my_tiles(k))
                    prefetch_l2_bulk(a.p[k].sched + (blockIdx.x + (long long)i * G) * a.tile_words,
                                     (uint32_t)(a.tile_words * 4));
            };
            prefetch_one(0, 0);
            prefetch_one(0, 1);
            int j = 0;
            for (int k = 0; k < 3; ++k) {
                const TlcPassCfg& pc = a.p[k];
                const int nt = my_tiles(k);
                if (k > 0) {
                    // poll the grid counter only once this CTA has arrived (pdone[k - 1] was
                    // waited on at the end of pass k - 1; polling one L2 line from every SM
                    // during the whole pass slows the pass's own traffic)
                    while (ld_acquire_gpu(&a.sync[k - 1]) < (unsigned long long)G) __nanosleep(32);
                    fence_proxy_async_global();
                    stamp(tr, 1 + 4 * k);
                }
                for (int i = 0; i < nt; ++i, ++j) {
                    const long long t = blockIdx.x + (long long)i * G;
                    const int s = j % NA;
                    if (j >= NA) mbar_wait(&R.aempty[s], (uint32_t)(j / NA - 1) & 1u);
                    fence_proxy_async();       // permuters' generic reads of the slot -> TMA write
                    mbar_arrive_expect_tx(&R.afull[s], (uint32_t)HL * 4u);
                    bulk_g2s(R.A + (size_t)s * HL, pc.in + t * HL, (uint32_t)HL * 4u, &R.afull[s]);
                    if (k == 0) {
                        prefetch_one(0, i + 2);
                        if (i + 1 == NA)       // pass-0 input tiles beyond the ring: into L2 now
                            for (int q = NA; q < nt; ++q)
                                prefetch_l2_bulk(pc.in + (blockIdx.x + (long long)q * G) * HL, (uint32_t)HL * 4u);
                    }
                }
                if (k < 2) {
                    // pass k + 1's schedules once this CTA's pass-k stores are complete: HBM is
                    // then free of this CTA's pass-k traffic, and the prefetch overlaps the barrier
                    mbar_wait_sleepy(&pdone[k], 0, 200);
                    for (int i = 0; i < my_tiles(k + 1); ++i) prefetch_one(k + 1, i);
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ---------------- storer
            int j = 0;
            int prev = -1;                   // B slot of the previous, not yet released store
            for (int k = 0; k < 3; ++k) {
                const TlcPassCfg& pc = a.p[k];
                const CUtensorMap* map = pc.kind == 2 ? &map_x2 : &map_x1;
                const int nt = my_tiles(k);
                for (int i = 0; i < nt; ++i, ++j) {
                    const long long t = blockIdx.x + (long long)i * G;
                    const int s = j % NB;
                    mbar_wait(&R.bfull[s], (uint32_t)(j / NB) & 1u);
                    tlc_store(pc.kind, map, pc.out, R.B + (size_t)s * HL, t, HL, pc.chunk, pc.nbox,
                              pc.box_outer, pc.box_words);
                    if (NB == 1) {
                        bulk_wait_read0();
                        mbar_arrive(&R.bempty[s]);
                    } else {
                        if (prev >= 0) {
                            bulk_wait_read1();       // the previous store has read its slot
                            mbar_arrive(&R.bempty[prev]);
                        }
                        prev = s;
                    }
                }
                if (k < 2) {
                    bulk_wait0();                    // this CTA's pass-k output is written
                    if (k == 0) stamp_if(tr, true, 14);
                    if (prev >= 0) {
                        mbar_arrive(&R.bempty[prev]);
                        prev = -1;
                    }
                    fence_proxy_async_global();      // async-proxy writes -> the generic release
                    if (k == 0) stamp_if(tr, true, 13);
                    red_relaxed_gpu_add(&a.sync[k], 1ull);
                    mbar_arrive(&pdone[k]);
                    stamp_if(tr, true, 4 + 4 * k);
                }
            }
            bulk_wait0();
        }
    } else {
        // ---------------- permuters
        // One flat sequence of this CTA's tiles over the three passes (j -> pass k, tile i):
        // schedule words are loaded AHEAD tiles ahead, across pass boundaries (they do not
        // depend on the data), into NBUF register buffers rotated by unrolling.
        const bool lead = tid == 64;
        const int nt0 = my_tiles(0), nt1 = my_tiles(1), nt2 = my_tiles(2);
        const int J = nt0 + nt1 + nt2;
        const uint64_t pol_first = policy_evict_first();
        constexpr int AHEAD = NWORDS <= 12 ? 2 : 1;
        constexpr int NBUF = AHEAD + 1;
        auto locate = [&](int jj, int& k, int& i) {
            k = jj < nt0 ? 0 : (jj < nt0 + nt1 ? 1 : 2);
            i = jj - (k == 0 ? 0 : (k == 1 ? nt0 : nt0 + nt1));
        };
        uint32_t wq[NBUF][NWORDS];
        auto load_words = [&](int jj, uint32_t* dstw) {
            int k, i;
            locate(jj, k, i);
            const uint32_t* sp = a.p[k].sched + (blockIdx.x + (long long)i * G) * a.tile_words +
                                 (warp - 2) * NWORDS * 32 + lane;
#pragma unroll
            for (int w = 0; w < NWORDS; ++w) dstw[w] = ld_nc_hint(sp + w * 32, pol_first);
        };
#pragma unroll
        for (int q = 0; q < AHEAD; ++q)
            if (q < J) load_words(q, wq[q]);
        int s = 0, sb = 0;
        uint32_t pa = 0u, pb = 1u;
        for (int j0 = 0; j0 < J; j0 += NBUF) {
#pragma unroll
            for (int u = 0; u < NBUF; ++u) {
                const int jj = j0 + u;
                if (jj >= J) break;
                int k, i;
                locate(jj, k, i);
                const TlcPassCfg& pc = a.p[k];
                mbar_wait(&R.afull[s], pa);
                if (i == 0) stamp_if(tr, lead, 2 + 4 * k);
                uint32_t* const Bs = R.B + (size_t)sb * HL;
                const uint32_t* const As = R.A + (size_t)s * HL;
                uint64_t* const bw = jj >= NB ? &R.bempty[sb] : nullptr;
                if constexpr (E == 2 * cilog2(HL) - 5) {
                    tlc_permute<EPT, E, TLC_FULL>(As, Bs, wq[u], pc.dec, 0u, &R.aempty[s], bw, pb, lane);
                } else {
                    const int kind = pc.kind == 1 ? TLC_X1 : (pc.kind == 2 ? TLC_X2 : TLC_ROWS);
                    const uint32_t lc = tlc_lane_const(kind, pc.dec, lane);
                    if (kind == TLC_X1)
                        tlc_permute<EPT, E, TLC_X1>(As, Bs, wq[u], pc.dec, lc, &R.aempty[s], bw, pb, lane);
                    else if (kind == TLC_X2)
                        tlc_permute<EPT, E, TLC_X2>(As, Bs, wq[u], pc.dec, lc, &R.aempty[s], bw, pb, lane);
                    else
                        tlc_permute<EPT, E, TLC_ROWS>(As, Bs, wq[u], pc.dec, lc, &R.aempty[s], bw, pb, lane);
                }
                mbar_arrive(&R.bfull[sb]);
                // look-ahead AFTER the permute's proxy fence (MEMBAR.CTA waits for every
                // outstanding load of the thread; across a pass boundary the next pass's words
                // come from HBM and would stall the last tiles of the pass)
                if (jj + AHEAD < J) load_words(jj + AHEAD, wq[(u + AHEAD) % NBUF]);
                if (i == (k == 0 ? nt0 : (k == 1 ? nt1 : nt2)) - 1) stamp_if(tr, lead, 3 + 4 * k);
                if (++s == NA) { s = 0; pa ^= 1u; }
                if (++sb == NB) { sb = 0; pb ^= 1u; }
            }
        }
    }
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        const unsigned long long old = atomicAdd(&a.sync[2], 1ull);
        if (old == (unsigned long long)G - 1) {
            a.sync[0] = 0;
            a.sync[1] = 0;
            a.sync[2] = 0;
            __threadfence();
        }
    }
    stamp(tr, 15);
}

// ------------------------------------------------------------------ cluster path (n = 2^15..2^18)

__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_size() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
// split cluster barrier: every thread of every block of the cluster arrives (release)
// and later waits (acquire); work between the two halves overlaps the barrier
__device__ __forceinline__ void cluster_arrive() {
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
}
// arrive without release semantics: for barriers whose only job is to order async-proxy
// (bulk copy) completions that every block has already observed on its own mbarrier
__device__ __forceinline__ void cluster_arrive_relaxed() {
    asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() {
    asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cta address -> the same offset in block `rank` of the cluster (shared::cluster)
__device__ __forceinline__ uint32_t map_to(uint32_t cta_addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(cta_addr), "r"(rank));
    return r;
}
// bulk copy of `bytes` from this block's shared memory to block `dst`'s (DSMEM), completion
// (complete_tx) on the destination block's mbarrier
__device__ __forceinline__ void bulk_s2cluster(uint32_t dst_cl, const void* src, uint32_t bytes, uint32_t mbar_cl) {
    asm volatile(
        "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst_cl),
        "r"(smem_u32(src)), "r"(bytes), "r"(mbar_cl)
        : "memory");
}

// One block's tile-coloured permute B[dst] = A[src] (full entry format):
// warp-round m of warp `warp`: lane x reads A[32*sigma + x] (bank x) and writes B[dst];
// the 32 dst of a round lie in 32 distinct banks (the tile colouring).
// With `self` (a block index) the destinations in send block `self` go straight to `Bself`
// (the buffer that block's exchange would have delivered them to: no copy to oneself);
// B and Bself are 128-byte aligned, so a destination keeps its bank either way.
template <int EPT, int LOGS>
__device__ __forceinline__ void block_permute(const uint32_t* __restrict__ A, uint32_t* __restrict__ B,
                                              const uint32_t* wc, int lane, uint32_t* Bself = nullptr,
                                              uint32_t self = 0, int logBw = 0) {
    constexpr int E = 2 * LOGS - 5;
    constexpr uint32_t EMASK = (1u << E) - 1u;
    constexpr uint32_t TMASK = (1u << LOGS) - 1u;
    uint32_t v[EPT], d[EPT];
#pragma unroll
    for (int m = 0; m < EPT; ++m) {
        const int bit = m * E, w = bit >> 5, off = bit & 31;
        uint32_t e;
        if (off + E <= 32) e = (wc[w] >> off) & EMASK;
        else e = __funnelshift_r(wc[w], wc[w + 1], off) & EMASK;
        v[m] = A[((e >> LOGS) << 5) | (uint32_t)lane];
        d[m] = e & TMASK;
    }
    if (Bself) {
#pragma unroll
        for (int m = 0; m < EPT; ++m) ((d[m] >> logBw) == self ? Bself : B)[d[m]] = v[m];
    } else {
#pragma unroll
        for (int m = 0; m < EPT; ++m) B[d[m]] = v[m];
    }
}

struct ClusterArgs {
    const uint32_t* in;
    uint32_t* out;
    const uint32_t* sched[3];
    long long tile_words;        // schedule words of one block's share of a phase
    unsigned long long* trace;   // optional %globaltimer stamps [block][16]
};

// Thm 9 (L537-L539) in ONE launch for arrays that fit in one cluster's shared memory
// (NEXT-4; the single-SM permutation of the prior work, here spread over
// the C <= 16 SMs of a cluster). Block g: three buffers of S words (buf0, buf1, buf2)
// and three mbarriers. Phase 1 buf0 -> buf1 (send blocks); exchange 1: send block q ->
// block q's buf2 at [g*Bw, ...) (DSMEM bulk copies, completion counted on block q's
// mbarrier); phase 2 buf2 -> buf0; exchange 2: buf0 -> block q's buf1 (free once every
// block has received exchange 1: split cluster barrier); phase 3 buf1 -> buf2 -> b.
// Every permute hop is conflict-free in both banks (tile colouring).
template <int EPT>
__global__ void __launch_bounds__(kTlcPerm, 1) cluster_kernel(const ClusterArgs a) {
    constexpr int S = kTlcPerm * EPT;
    constexpr int LOGS = cilog2(S);
    constexpr int E = 2 * LOGS - 5;
    constexpr int NWORDS = (EPT * E + 31) / 32;
    constexpr int TW = (kTlcPerm / 32) * NWORDS * 32;              // schedule words per block and phase
    // up to 8192 words per block the three phases' schedules ride in shared memory (one TMA
    // round trip with a); beyond, they are read from global memory (L2-prefetched)
    constexpr bool SMEM_SCHED = EPT <= 16;
    extern __shared__ __align__(128) uint32_t smem[];
    uint32_t* buf0 = smem;
    uint32_t* buf1 = smem + S;
    uint32_t* buf2 = smem + 2 * S;
    uint32_t* sch = smem + 3 * S;                                   // [3][TW] when SMEM_SCHED
    // [0] a (+ phase-1 schedule), [1] exchange 1, [2] exchange 2, [3] phases 2-3 schedules
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem + 3 * S + (SMEM_SCHED ? 3 * TW : 0));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t g = cluster_rank(), C = cluster_size();
    const uint32_t Bw = (uint32_t)S / C;                          // words per exchanged block
    const int logBw = 31 - __clz((int)Bw);
    const uint32_t rx_bytes = ((uint32_t)S - Bw) * 4u;            // received from the C-1 peers
    if (tid == 0) {
        for (int i = 0; i < 4; ++i) mbar_init(&bar[i], 1);
        fence_mbar_init();
        // every byte this block will receive is announced before any peer can send
        mbar_arrive_expect_tx(&bar[1], rx_bytes);
        mbar_arrive_expect_tx(&bar[2], rx_bytes);
        if constexpr (SMEM_SCHED) {
            mbar_arrive_expect_tx(&bar[0], (uint32_t)(S + TW) * 4u);
            bulk_g2s(buf0, a.in + (size_t)g * S, (uint32_t)S * 4u, &bar[0]);
            bulk_g2s(sch, a.sched[0] + (size_t)g * TW, (uint32_t)TW * 4u, &bar[0]);
            mbar_arrive_expect_tx(&bar[3], (uint32_t)(2 * TW) * 4u);
            bulk_g2s(sch + TW, a.sched[1] + (size_t)g * TW, (uint32_t)TW * 4u, &bar[3]);
            bulk_g2s(sch + 2 * TW, a.sched[2] + (size_t)g * TW, (uint32_t)TW * 4u, &bar[3]);
        } else {
            mbar_arrive_expect_tx(&bar[0], (uint32_t)S * 4u);
            bulk_g2s(buf0, a.in + (size_t)g * S, (uint32_t)S * 4u, &bar[0]);
            // phases 2 and 3 read their schedules after the exchanges: pull them into L2 now,
            // in the same HBM round trip as a and phase 1's schedule
            for (int f = 1; f < 3; ++f) prefetch_l2_bulk(a.sched[f] + (size_t)g * TW, (uint32_t)TW * 4u);
        }
    }
    __syncthreads();
    stamp(a.trace, 0);
    cluster_arrive();                       // (A) mbarriers initialised and armed
    uint32_t wc[NWORDS];
    // lane's schedule words of phase f: coalesced (word w of lane x at (warp*NWORDS + w)*32 + x)
    auto load_sched = [&](int f) {
        if constexpr (SMEM_SCHED) {
            const uint32_t* sp = sch + f * TW + warp * NWORDS * 32 + lane;
#pragma unroll
            for (int w = 0; w < NWORDS; ++w) wc[w] = sp[w * 32];
        } else {
            const uint32_t* sp = a.sched[f] + (size_t)g * TW + warp * NWORDS * 32 + lane;
#pragma unroll
            for (int w = 0; w < NWORDS; ++w) wc[w] = __ldg(sp + w * 32);
        }
    };
    if constexpr (!SMEM_SCHED) load_sched(0);
    mbar_wait(&bar[0], 0);
    stamp(a.trace, 1);
    if constexpr (SMEM_SCHED) load_sched(0);
    block_permute<EPT, LOGS>(buf0, buf1, wc, lane, buf2, g, logBw);   // phase 1 (own block -> buf2)
    fence_proxy_async();                    // generic writes of buf1 -> the bulk copies' reads
    if constexpr (!SMEM_SCHED) load_sched(1);
    __syncthreads();
    stamp(a.trace, 2);
    cluster_wait();                         // (A): every peer's mbarriers are armed
    stamp(a.trace, 3);
    if (tid == 0) {
        const uint32_t dst0 = smem_u32(buf2 + g * Bw), mb = smem_u32(&bar[1]);
        for (uint32_t q = 0; q < C; ++q)
            if (q != g) bulk_s2cluster(map_to(dst0, q), buf1 + q * Bw, Bw * 4u, map_to(mb, q));
    }
    if constexpr (SMEM_SCHED) {
        mbar_wait(&bar[3], 0);
        load_sched(1);
    }
    mbar_wait(&bar[1], 0);                  // exchange 1 landed in buf2
    stamp(a.trace, 4);
    // (B) exchange 1 into me is complete. Passing (B) tells a block that every exchange-1
    // copy (hence every read out of its buf1) has completed: completions each block observed
    // on its own mbarrier (complete_tx), so no release of generic writes is needed here
    cluster_arrive_relaxed();
    block_permute<EPT, LOGS>(buf2, buf0, wc, lane, buf1, g, logBw);   // phase 2 (own block -> buf1)
    fence_proxy_async();
    load_sched(2);
    __syncthreads();
    stamp(a.trace, 5);
    cluster_wait();                         // (B): every block received exchange 1 -> every buf1 is free
    stamp(a.trace, 6);
    if (tid == 0) {
        const uint32_t dst0 = smem_u32(buf1 + g * Bw), mb = smem_u32(&bar[2]);
        for (uint32_t q = 0; q < C; ++q)
            if (q != g) bulk_s2cluster(map_to(dst0, q), buf0 + q * Bw, Bw * 4u, map_to(mb, q));
    }
    mbar_wait(&bar[2], 0);                  // exchange 2 landed in buf1
    stamp(a.trace, 7);
    cluster_arrive_relaxed();               // (C) exchange 2 into me is complete (lifetime only)
    block_permute<EPT, LOGS>(buf1, buf2, wc, lane);               // phase 3
    fence_proxy_async();
    __syncthreads();
    if (tid == 0) {
        stamp(a.trace, 8);
        bulk_s2g(a.out + (size_t)g * S, buf2, (uint32_t)S * 4u);
        bulk_commit();
        bulk_wait_read0();
        stamp(a.trace, 9);
    }
    cluster_wait();                         // (C): no peer still reads my buf0 before I exit
    stamp(a.trace, 10);
}

// ------------------------------------------------------------------ transpose

// PAPER.md §V (Lemma 5): w x w tiles through shared memory. The tile is stored
// with row stride 33, i.e. element (i, j) in bank (i + j) mod 32 — the diagonal
// arrangement of Fig. 4 — so both the row-wise write and the column-wise read
// are conflict-free.
__global__ void __launch_bounds__(256) transpose_kernel(const uint32_t* __restrict__ in,
                                                        uint32_t* __restrict__ out, int logr,
                                                        int logc) {
    __shared__ uint32_t tile[32][33];
    const long long rows = 1ll << logr, cols = 1ll << logc;
    const int tx = threadIdx.x, ty = threadIdx.y;
    const long long bx = blockIdx.x, by = blockIdx.y;
    pdl_wait();
#pragma unroll
    for (int j = 0; j < 32; j += 8)
        tile[ty + j][tx] = __ldg(in + (by * 32 + ty + j) * cols + bx * 32 + tx);
    __syncthreads();
    pdl_launch_dependents();
#pragma unroll
    for (int j = 0; j < 32; j += 8) out[(bx * 32 + ty + j) * rows + by * 32 + tx] = tile[tx][ty + j];
}

// 64 x 64 tiles with 128-bit global loads and stores (16 KiB per CTA, 8 CTAs per
// SM: 128 KiB of loads in flight per SM, what HBM3e needs to stay busy). In
// shared memory, row r keeps its 16-byte chunks XOR-swizzled: chunk c4 of row r
// sits at chunk c4 ^ ((r >> 2) & 7). The 128-bit row writes stay conflict-free
// (a quarter-warp covers 8 distinct chunks of one row) and so do the column
// reads: lane (il, jl) reads row 4*(8*ih + il) + q, column 4*jh + jl, bank
// ((jh ^ il) & 7)*4 + jl -- 32 distinct banks, the role Fig. 4's diagonal
// arrangement plays for the paper's w x w tiles. Each lane gathers four rows of
// one column into a uint4, so 8 lanes store 128 contiguous bytes of an output row.
__global__ void __launch_bounds__(256) transpose64_kernel(const uint32_t* __restrict__ in,
                                                          uint32_t* __restrict__ out, int logr,
                                                          int logc) {
    __shared__ __align__(16) uint32_t tile[64 * 64];
    const long long rows = 1ll << logr, cols = 1ll << logc;
    const int tid = threadIdx.x;
    const long long bx = blockIdx.x, by = blockIdx.y;     // column tile, row tile
    pdl_wait();
    uint4 v[4];
#pragma unroll
    for (int it = 0; it < 4; ++it) {
        const int idx = tid + 256 * it, r = idx >> 4, c4 = idx & 15;
        v[it] = ld_nc_v4(in + (by * 64 + r) * cols + bx * 64 + c4 * 4);
    }
#pragma unroll
    for (int it = 0; it < 4; ++it) {
        const int idx = tid + 256 * it, r = idx >> 4, c4 = idx & 15;
        *reinterpret_cast<uint4*>(tile + r * 64 + ((c4 ^ ((r >> 2) & 7)) << 2)) = v[it];
    }
    __syncthreads();
    pdl_launch_dependents();
#pragma unroll
    for (int it = 0; it < 4; ++it) {
        const int idx = tid + 256 * it;
        const int il = idx & 7, jl = (idx >> 3) & 3, ih = (idx >> 5) & 1, jh = idx >> 6;
        const int i4 = ih * 8 + il, j = jh * 4 + jl;
        const int col = (jh ^ il) * 4 + jl;   // swizzled word of column j (il < 8)
        uint4 w;
        w.x = tile[(4 * i4 + 0) * 64 + col];
        w.y = tile[(4 * i4 + 1) * 64 + col];
        w.z = tile[(4 * i4 + 2) * 64 + col];
        w.w = tile[(4 * i4 + 3) * 64 + col];
        st_v4(out + (bx * 64 + j) * rows + by * 64 + i4 * 4, w);
    }
}

// ------------------------------------------------------------------ comparators

// D-designated (L365): coalesced 128-bit reads of p and a, casual writes of b.
__global__ void __launch_bounds__(256) scatter_kernel(const int32_t* __restrict__ p,
                                                      const uint32_t* __restrict__ a,
                                                      uint32_t* __restrict__ b, long long nv) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv;
         v += (long long)gridDim.x * blockDim.x) {
        const uint4 pv = ld_nc_v4(reinterpret_cast<const uint32_t*>(p) + 4 * v);
        const uint4 av = ld_nc_v4(a + 4 * v);
        b[pv.x] = av.x;
        b[pv.y] = av.y;
        b[pv.z] = av.z;
        b[pv.w] = av.w;
    }
}

// S-designated (L373): coalesced reads of q, casual reads of a, coalesced writes of b.
__global__ void __launch_bounds__(256) gather_kernel(const int32_t* __restrict__ q,
                                                     const uint32_t* __restrict__ a,
                                                     uint32_t* __restrict__ b, long long nv) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv;
         v += (long long)gridDim.x * blockDim.x) {
        const uint4 qv = ld_nc_v4(reinterpret_cast<const uint32_t*>(q) + 4 * v);
        uint4 o;
        o.x = __ldg(a + qv.x);
        o.y = __ldg(a + qv.y);
        o.z = __ldg(a + qv.z);
        o.w = __ldg(a + qv.w);
        st_v4(b + 4 * v, o);
    }
}

// 8-byte element variants (Table II(b)): 2 x 64-bit element loads per 128-bit p/q load
__global__ void __launch_bounds__(256) scatter64_kernel(const int32_t* __restrict__ p,
                                                        const uint2* __restrict__ a,
                                                        uint2* __restrict__ b, long long nv) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv;
         v += (long long)gridDim.x * blockDim.x) {
        const uint4 pv = ld_nc_v4(reinterpret_cast<const uint32_t*>(p) + 4 * v);
        const uint4 a0 = ld_nc_v4(reinterpret_cast<const uint32_t*>(a + 4 * v));
        const uint4 a1 = ld_nc_v4(reinterpret_cast<const uint32_t*>(a + 4 * v + 2));
        b[pv.x] = make_uint2(a0.x, a0.y);
        b[pv.y] = make_uint2(a0.z, a0.w);
        b[pv.z] = make_uint2(a1.x, a1.y);
        b[pv.w] = make_uint2(a1.z, a1.w);
    }
}

__global__ void __launch_bounds__(256) gather64_kernel(const int32_t* __restrict__ q,
                                                       const uint2* __restrict__ a,
                                                       uint2* __restrict__ b, long long nv) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv;
         v += (long long)gridDim.x * blockDim.x) {
        const uint4 qv = ld_nc_v4(reinterpret_cast<const uint32_t*>(q) + 4 * v);
        const uint2 x0 = __ldg(a + qv.x), x1 = __ldg(a + qv.y), x2 = __ldg(a + qv.z), x3 = __ldg(a + qv.w);
        st_v4(reinterpret_cast<uint32_t*>(b + 4 * v), make_uint4(x0.x, x0.y, x1.x, x1.y));
        st_v4(reinterpret_cast<uint32_t*>(b + 4 * v + 2), make_uint4(x2.x, x2.y, x3.x, x3.y));
    }
}

// Block gather for P that moves whole aligned 32-word blocks in order (D_w(P) = n/w with
// p[32j + x] = 32 g + x): qb[g] = j, one index per 32 words; each thread moves 16 bytes,
// 8 consecutive threads one 128-byte block (full-line reads and writes).
__global__ void __launch_bounds__(256) block_gather_kernel(const int32_t* __restrict__ qb,
                                                           const uint32_t* __restrict__ a,
                                                           uint32_t* __restrict__ b, long long nv) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv;
         v += (long long)gridDim.x * blockDim.x) {
        const long long src = (long long)__ldg(qb + (v >> 3)) * 8 + (v & 7);
        st_v4(b + 4 * v, ld_nc_v4(a + 4 * src));
    }
}

__global__ void __launch_bounds__(256) copy_kernel(const uint32_t* __restrict__ a,
                                                   uint32_t* __restrict__ b, long long nv) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv;
         v += (long long)gridDim.x * blockDim.x)
        st_v4(b + 4 * v, ld_nc_v4(a + 4 * v));
}

int ilog2i(long long v) {
    int k = 0;
    while ((1ll << k) < v) ++k;
    return k;
}

int sm_count() {
    static int count = 0;
    if (!count) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&count, cudaDevAttrMultiProcessorCount, dev);
        if (count <= 0) count = 148;
    }
    return count;
}

template <typename K, typename... Args>
cudaError_t launch(K kernel, dim3 grid, dim3 block, size_t smem, cudaStream_t s, bool pdl,
                   Args... args) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, args...);
}

size_t fused_smem(const HostPlan& P) { return (size_t)P.r * P.fused_Ls * 4; }
size_t row_smem(const HostPlan& P, int f) { return (size_t)P.rp[f].h * P.rp[f].Ls * 4; }

Io make_io(const IoMode& m) {
    Io o{};
    o.cross = m.cross;
    o.logw = m.cross ? 0 : ilog2i(m.w);
    o.logBP = m.cross ? ilog2i(m.blockP) : 0;
    o.strideK = m.strideK;
    o.strideP = m.strideP;
    o.cta_stride = m.cta_stride;
    return o;
}

template <typename K>
cudaError_t set_smem(K kernel, size_t bytes) {
    cudaError_t e = cudaFuncSetAttribute((const void*)kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute((const void*)kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                                 100);
    return e;
}

size_t tma_smem(const HostPlan& P, int f) {
    const RowPass& rp = P.rp[f];
    const PhaseGeom& g = P.ph[rp.phase];
    if (rp.split && rp.split_stg)
        return g.dense ? (size_t)3 * (g.L / 2) * 4 + (size_t)5 * kStgDenseWords * 4 + (3 + 2 * 5) * 8
                       : (size_t)3 * (g.L / 2) * 4 + (size_t)4 * kStgChunkWords * 4 + (3 + 2 * 4) * 8;
    if (rp.split) return (size_t)3 * (g.L / 2) * 4 + 3 * 8;
    const size_t stage = (size_t)rp.h * rp.Ls * 4 + (rp.sg ? 0 : (size_t)rp.h * g.wpl * 4);
    return rp.stages * stage + rp.stages * 8;
}

template <int EPT>
const void* split_kernel_ptr(bool dense) {
    if constexpr (EPT < 8) {
        return nullptr;
    } else {
        return dense ? (const void*)row_pass_split_kernel<EPT, true, false>
                     : (const void*)row_pass_split_kernel<EPT, false, false>;
    }
}

template <int EPT>
const void* tma_kernel_ptr(bool cross, bool sg, bool split = false, bool dense = false, bool keep = true,
                           bool stg = false) {
    if constexpr (EPT == 32 || EPT == 64) {
        if (split && stg) return dense ? (const void*)row_pass_split_stg_kernel<EPT, true>
                                       : (const void*)row_pass_split_stg_kernel<EPT, false>;
    }
    if (split) return split_kernel_ptr<EPT>(dense);
    if (sg) return cross ? (const void*)row_pass_tma_kernel<EPT, true, true>
                         : (const void*)row_pass_tma_kernel<EPT, false, true>;
    return cross ? (const void*)row_pass_tma_kernel<EPT, true> : (const void*)row_pass_tma_kernel<EPT, false>;
}

template <int EPT>
cudaError_t set_tma_smem(bool cross, size_t smem) {
    cudaError_t e = set_smem(tma_kernel_ptr<EPT>(cross, false), smem);
    if (e == cudaSuccess) e = set_smem(tma_kernel_ptr<EPT>(cross, true), smem);
    if constexpr (EPT >= 8) {
        for (int v = 0; v < 2 && e == cudaSuccess; ++v)
            e = set_smem(tma_kernel_ptr<EPT>(cross, true, true, v & 1), smem);
    }
    if constexpr (EPT == 32 || EPT == 64) {
        if (e == cudaSuccess) e = set_smem(tma_kernel_ptr<EPT>(cross, true, true, false, false, true), smem);
        if (e == cudaSuccess) e = set_smem(tma_kernel_ptr<EPT>(cross, true, true, true, false, true), smem);
    }
    return e;
}

template <int EPT>
cudaError_t grid_tma(HostPlan& P, int f) {
    RowPass& rp = P.rp[f];
    const size_t smem = tma_smem(P, f);
    int nb = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
        &nb, tma_kernel_ptr<EPT>(rp.out.cross != 0, rp.sg != 0, rp.split != 0, P.ph[rp.phase].dense != 0,
                                 rp.split_keep != 0, rp.split_stg != 0),
        rp.threads, smem);
    if (e != cudaSuccess) return e;
    if (nb < 1) return cudaErrorInvalidConfiguration;
    const long long cap = (long long)nb * sm_count();
    rp.grid = rp.ctas < cap ? rp.ctas : cap;
    return cudaSuccess;
}

size_t tlc_smem(const HostPlan& P, int f) {
    const TlcPass& tp = P.tp[f];
    // + 2 mbarriers of the fused kernel (pass k stored by this CTA)
    return (size_t)(tp.stages + tp.bslots) * tp.HL * 4 + (size_t)(tp.stages + tp.bslots) * 8 * 2 + 16;
}

// Calls f(EPT, E) (std::integral_constant) for the compiled (elements per thread,
// entry bits) pairs of the TLC kernels: the full formats 2*log2(512*EPT) - 5 and
// the compact widths of plan.hpp tlc_compact_supported().
template <class F>
cudaError_t tlc_dispatch(int ept, int E, F&& f) {
    using std::integral_constant;
    if (ept == 8 && E == 19) return f(integral_constant<int, 8>{}, integral_constant<int, 19>{});
    if (ept == 16) {
        switch (E) {
            case 21: return f(integral_constant<int, 16>{}, integral_constant<int, 21>{});
            case 20: return f(integral_constant<int, 16>{}, integral_constant<int, 20>{});
            case 19: return f(integral_constant<int, 16>{}, integral_constant<int, 19>{});
            case 18: return f(integral_constant<int, 16>{}, integral_constant<int, 18>{});
            case 17: return f(integral_constant<int, 16>{}, integral_constant<int, 17>{});
            case 16: return f(integral_constant<int, 16>{}, integral_constant<int, 16>{});
            case 15: return f(integral_constant<int, 16>{}, integral_constant<int, 15>{});
        }
    }
    if (ept == 32 && E == 23) return f(integral_constant<int, 32>{}, integral_constant<int, 23>{});
    if (ept == 32 && E == 22) return f(integral_constant<int, 32>{}, integral_constant<int, 22>{});
    if (ept == 32 && E == 21) return f(integral_constant<int, 32>{}, integral_constant<int, 21>{});
    return cudaErrorInvalidValue;
}

template <class K>
cudaError_t prep_tlc_kernel(K kernel, size_t smem, long long ntiles, long long& grid) {
    cudaError_t e = set_smem(kernel, smem);
    if (e != cudaSuccess) return e;
    int nb = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kernel, 64 + kTlcPerm, smem);
    if (e != cudaSuccess) return e;
    if (nb < 1) return cudaErrorInvalidConfiguration;
    const long long cap = (long long)nb * sm_count();
    grid = ntiles < cap ? ntiles : cap;
    return cudaSuccess;
}

cudaError_t prep_tlc(HostPlan& P) {
    if (P.fused3) {
        return tlc_dispatch(P.tp[0].ept, P.tp[0].E, [&](auto ept, auto E) {
            long long g = 0;
            const cudaError_t e = prep_tlc_kernel(fused_tlc_kernel<ept, E>, tlc_smem(P, 0), 1, g);
            P.fused3_grid = sm_count();      // one co-resident CTA per SM (grid barriers)
            return e;
        });
    }
    cudaError_t e = cudaSuccess;
    for (int f = 0; f < 3 && e == cudaSuccess; ++f) {
        TlcPass& tp = P.tp[f];
        long long g = 0;
        e = tlc_dispatch(tp.ept, tp.E, [&](auto ept, auto E) {
            const size_t smem = tlc_smem(P, f);
            if (tp.out_kind == 0) return prep_tlc_kernel(row_pass_tlc_kernel<ept, 0, E>, smem, tp.ntiles, g);
            if (tp.out_kind == 1) return prep_tlc_kernel(row_pass_tlc_kernel<ept, 1, E>, smem, tp.ntiles, g);
            return prep_tlc_kernel(row_pass_tlc_kernel<ept, 2, E>, smem, tp.ntiles, g);
        });
        tp.grid = g;
        P.rp[f].grid = g;
    }
    return e;
}

}  // namespace

cudaError_t make_tlc_maps(const HostPlan& P, uint32_t* x1, uint32_t* x2, CUtensorMap* maps) {
    static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
    if (!encode) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
        if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn) return cudaErrorNotSupported;
        encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    }
    const cuuint64_t r = (cuuint64_t)P.r, c = (cuuint64_t)P.c;
    const cuuint64_t h1 = P.tp[0].h, h2 = P.tp[1].h, h3 = P.tp[2].h;
    // row-sharded plans: a rank's X1 holds its r/world rows, its X2 its c/world columns
    const cuuint64_t rX1 = P.r_l ? (cuuint64_t)P.r_l : r, cX2 = P.c_l ? (cuuint64_t)P.c_l : c;
    std::memset(maps, 0, 3 * sizeof(CUtensorMap));
    // Maps whose box rows are a tile's contiguous chunks (64 bytes at h1*h2 = 16 words; at
    // most 256 words per row): a 16-byte innermost box dimension makes the TMA unit emit
    // 16-byte rows (measured 1.5x slower per pass, scripts/micro/tile_io.py).
    //   X1 = [K][i][k_in]: K-blocks of r*h2 words; pass-1 tile t writes [t*h1*h2, +h1*h2) of each
    //   X2 = [I'][K][i_in'][k_in]: I'-blocks of c*h3 words; pass-2 tile K writes [K*h3*h2, +h3*h2)
    const cuuint64_t ch[2] = {h1 * h2, h3 * h2};
    const cuuint64_t blk[2] = {rX1 * h2, cX2 * h3};
    const cuuint64_t nblk[2] = {c / h2, r / h3};
    void* base[2] = {x1, x2};
    for (int m = 0; m < 2; ++m) {
        const cuuint64_t rw = std::min<cuuint64_t>(ch[m], 256);
        const cuuint64_t dims[3] = {rw, blk[m] / rw, nblk[m]};
        const cuuint64_t strides[2] = {rw * 4, blk[m] * 4};
        const cuuint32_t box[3] = {(cuuint32_t)rw, (cuuint32_t)(ch[m] / rw),
                                   (cuuint32_t)std::min<cuuint64_t>(256, nblk[m])};
        const cuuint32_t es[3] = {1, 1, 1};
        if (encode(&maps[m], CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, base[m], dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return cudaErrorInvalidValue;
    }
    return cudaSuccess;
}

cudaError_t launch_tlc_pass(const HostPlan& P, int f, const CUtensorMap* maps, const uint32_t* sched,
                            const uint32_t* in, uint32_t* out, cudaStream_t s, bool pdl,
                            unsigned long long* trace) {
    const TlcPass& tp = P.tp[f];
    TlcArgs ta{};
    ta.in = in;
    ta.out = out;
    ta.sched = sched;
    ta.ntiles = (int)tp.ntiles;
    ta.na = tp.stages;
    ta.nb = tp.bslots;
    ta.tile_words = tp.tile_words;
    ta.trace = trace;
    ta.prefetch_in = (f == 0) ? 1 : 0;   // pass 1 reads `a` from HBM; later passes read L2-resident X
    ta.segs = tp.segs;
    ta.seg_len = tp.seg_len;
    ta.seg_stride = tp.seg_stride;
    const long long h1 = P.tp[0].h, h2 = P.tp[1].h, h3 = P.tp[2].h;
    if (tp.out_kind == 1) {
        const long long outer = P.c / h2, bo = outer < 256 ? outer : 256;
        ta.box_outer = (int)bo;
        ta.nbox = (int)(outer / bo);
        ta.box_words = (int)(bo * h1 * h2);
        ta.chunk = (int)(h1 * h2 / std::min<long long>(h1 * h2, 256));
    } else if (tp.out_kind == 2) {
        const long long outer = P.r / h3, bo = outer < 256 ? outer : 256;
        ta.box_outer = (int)bo;
        ta.nbox = (int)(outer / bo);
        ta.box_words = (int)(bo * h3 * h2);
        ta.chunk = (int)(h3 * h2 / std::min<long long>(h3 * h2, 256));
    }
    const CUtensorMap& map = maps[tp.out_kind == 2 ? 1 : 0];
    const dim3 grid((unsigned)tp.grid), block(64 + kTlcPerm);
    const size_t smem = tlc_smem(P, f);
    ta.dec = tp.dec;
    return tlc_dispatch(tp.ept, tp.E, [&](auto ept, auto E) {
        if (tp.out_kind == 0) return launch(row_pass_tlc_kernel<ept, 0, E>, grid, block, smem, s, pdl, map, ta);
        if (tp.out_kind == 1) return launch(row_pass_tlc_kernel<ept, 1, E>, grid, block, smem, s, pdl, map, ta);
        return launch(row_pass_tlc_kernel<ept, 2, E>, grid, block, smem, s, pdl, map, ta);
    });
}

cudaError_t launch_tlc_fused(const HostPlan& P, const CUtensorMap* maps, const uint32_t* const sched[3],
                             const uint32_t* a, uint32_t* x1, uint32_t* x2, uint32_t* b,
                             unsigned long long* sync, cudaStream_t s, unsigned long long* trace) {
    TlcFusedArgs fa{};
    const uint32_t* ins[3] = {a, x1, x2};
    uint32_t* outs[3] = {x1, x2, b};
    const long long h1 = P.tp[0].h, h2 = P.tp[1].h, h3 = P.tp[2].h;
    for (int f = 0; f < 3; ++f) {
        const TlcPass& tp = P.tp[f];
        TlcPassCfg& pc = fa.p[f];
        pc.in = ins[f];
        pc.out = outs[f];
        pc.sched = sched[f];
        pc.ntiles = (int)tp.ntiles;
        pc.kind = tp.out_kind;
        pc.dec = tp.dec;
        if (tp.out_kind == 1) {
            const long long outer = P.c / h2, bo = outer < 256 ? outer : 256;
            pc.box_outer = (int)bo;
            pc.nbox = (int)(outer / bo);
            pc.box_words = (int)(bo * h1 * h2);
            pc.chunk = (int)(h1 * h2 / std::min<long long>(h1 * h2, 256));
        } else if (tp.out_kind == 2) {
            const long long outer = P.r / h3, bo = outer < 256 ? outer : 256;
            pc.box_outer = (int)bo;
            pc.nbox = (int)(outer / bo);
            pc.box_words = (int)(bo * h3 * h2);
            pc.chunk = (int)(h3 * h2 / std::min<long long>(h3 * h2, 256));
        }
    }
    fa.tile_words = P.tp[0].tile_words;
    fa.na = P.tp[0].stages;
    fa.nb = P.tp[0].bslots;
    fa.sync = sync;
    fa.trace = trace;
    const dim3 grid((unsigned)P.fused3_grid), block(64 + kTlcPerm);
    const size_t smem = tlc_smem(P, 0);
    return tlc_dispatch(P.tp[0].ept, P.tp[0].E, [&](auto ept, auto E) {
        return launch(fused_tlc_kernel<ept, E>, grid, block, smem, s, false, maps[0], maps[1], fa);
    });
}

const void* cluster_kernel_ptr(int ept) {
    switch (ept) {
        case 4: return (const void*)cluster_kernel<4>;
        case 8: return (const void*)cluster_kernel<8>;
        case 16: return (const void*)cluster_kernel<16>;
        case 32: return (const void*)cluster_kernel<32>;
    }
    return nullptr;
}
size_t cluster_smem(const HostPlan& P) {
    // three S-word buffers, the three phases' schedules when a thread owns <= 16 elements,
    // four mbarriers (cluster_kernel)
    const TlcPass& tp = P.tp[0];
    return (size_t)3 * tp.HL * 4 + (tp.ept <= 16 ? (size_t)3 * tp.tile_words * 4 : 0) + 4 * 8;
}

cudaError_t launch_cluster(const HostPlan& P, const uint32_t* const sched[3], const uint32_t* a,
                           uint32_t* b, cudaStream_t s, unsigned long long* trace) {
    ClusterArgs ca{};
    ca.trace = trace;
    ca.in = a;
    ca.out = b;
    for (int f = 0; f < 3; ++f) ca.sched[f] = sched[f];
    ca.tile_words = P.tp[0].tile_words;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)P.cluster);
    cfg.blockDim = dim3(kTlcPerm);
    cfg.dynamicSmemBytes = cluster_smem(P);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)P.cluster;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    switch (P.tp[0].ept) {
        case 4: return cudaLaunchKernelEx(&cfg, cluster_kernel<4>, ca);
        case 8: return cudaLaunchKernelEx(&cfg, cluster_kernel<8>, ca);
        case 16: return cudaLaunchKernelEx(&cfg, cluster_kernel<16>, ca);
        case 32: return cudaLaunchKernelEx(&cfg, cluster_kernel<32>, ca);
    }
    return cudaErrorInvalidValue;
}

cudaError_t prepare_kernels(HostPlan& P) {
    if (P.direct) return cudaSuccess;     // one stream kernel, no attributes to set
    if (P.passes == 2) {
        const void* k = cluster_kernel_ptr(P.tp[0].ept);
        if (!k) return cudaErrorInvalidValue;
        cudaError_t e = set_smem(k, cluster_smem(P));
        if (e == cudaSuccess && P.cluster > 8)
            e = cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        return e;
    }
    if (P.layout == 3) return prep_tlc(P);
    cudaError_t e = cudaSuccess;
    auto set = [&](const void* k, size_t bytes) {
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    };
    if (P.passes == 1) {
        const size_t b = fused_smem(P);
        switch (P.fused_ept) {
            case 4: set((const void*)fused_kernel<4>, b); break;
            case 8: set((const void*)fused_kernel<8>, b); break;
            case 16: set((const void*)fused_kernel<16>, b); break;
            case 32: set((const void*)fused_kernel<32>, b); break;
            default: return cudaErrorInvalidValue;
        }
        return e;
    }
    // one attribute per template instance: use the largest request among the passes
    size_t need[7] = {0, 0, 0, 0, 0, 0, 0};        // plain kernel, index log2(ept)
    size_t need_t[2][7] = {{0}, {0}};              // TMA kernel [cross][log2(ept)]
    for (int f = 0; f < 3; ++f) {
        const int li = ilog2i(P.rp[f].ept);
        if (li < 2 || li > 6) return cudaErrorInvalidValue;
        if (P.rp[f].tma) {
            size_t& nt = need_t[P.rp[f].out.cross ? 1 : 0][li];
            nt = nt > tma_smem(P, f) ? nt : tma_smem(P, f);
        } else {
            need[li] = need[li] > row_smem(P, f) ? need[li] : row_smem(P, f);
        }
    }
    for (int cx = 0; cx < 2 && e == cudaSuccess; ++cx) {
        if (need_t[cx][2]) e = set_tma_smem<4>(cx, need_t[cx][2]);
        if (e == cudaSuccess && need_t[cx][3]) e = set_tma_smem<8>(cx, need_t[cx][3]);
        if (e == cudaSuccess && need_t[cx][4]) e = set_tma_smem<16>(cx, need_t[cx][4]);
        if (e == cudaSuccess && need_t[cx][5]) e = set_tma_smem<32>(cx, need_t[cx][5]);
        if (e == cudaSuccess && need_t[cx][6]) e = set_tma_smem<64>(cx, need_t[cx][6]);
    }
    for (int f = 0; f < 3 && e == cudaSuccess; ++f) {
        if (P.rp[f].tma != 1) continue;
        switch (P.rp[f].ept) {
            case 4: e = grid_tma<4>(P, f); break;
            case 8: e = grid_tma<8>(P, f); break;
            case 16: e = grid_tma<16>(P, f); break;
            case 32: e = grid_tma<32>(P, f); break;
            case 64: e = grid_tma<64>(P, f); break;
        }
    }
    if (e != cudaSuccess) return e;
    if (need[2]) set((const void*)row_pass_kernel<4>, need[2]);
    if (need[3]) set((const void*)row_pass_kernel<8>, need[3]);
    if (need[4]) set((const void*)row_pass_kernel<16>, need[4]);
    if (need[5]) set((const void*)row_pass_kernel<32>, need[5]);
    if (need[6]) set((const void*)row_pass_kernel<64>, need[6]);
    return e;
}

cudaError_t launch_fused(const HostPlan& P, const uint32_t* const sched[3], const uint32_t* a,
                         uint32_t* b, cudaStream_t s) {
    FusedArgs fa{};
    fa.in = a;
    fa.out = b;
    for (int f = 0; f < 3; ++f) {
        fa.sched[f] = sched[f];
        fa.E[f] = P.ph[f].E;
        fa.epw[f] = P.ph[f].epw;
        fa.w64[f] = P.ph[f].w64;
    }
    fa.logr = ilog2i(P.r);
    fa.logc = ilog2i(P.c);
    fa.Ls = P.fused_Ls;
    const dim3 grid(1), block(P.fused_threads);
    const size_t smem = fused_smem(P);
    switch (P.fused_ept) {
        case 4: return launch(fused_kernel<4>, grid, block, smem, s, false, fa);
        case 8: return launch(fused_kernel<8>, grid, block, smem, s, false, fa);
        case 16: return launch(fused_kernel<16>, grid, block, smem, s, false, fa);
        case 32: return launch(fused_kernel<32>, grid, block, smem, s, false, fa);
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_row_pass(const HostPlan& P, int f, const uint32_t* sched, const uint32_t* in,
                            uint32_t* out, cudaStream_t s, bool pdl, unsigned long long* trace,
                            const CUtensorMap* map) {
    const RowPass& rp = P.rp[f];
    const PhaseGeom& g = P.ph[rp.phase];
    RowArgs ra{};
    ra.trace = trace;
    ra.in = in;
    ra.out = out;
    ra.sched = sched;
    ra.logL = g.logL;
    ra.logh = ilog2i(rp.h);
    ra.Ls = rp.Ls;
    ra.E = g.E;
    ra.epw = g.epw;
    ra.w64 = g.w64;
    ra.dense = g.dense;
    ra.sched_words_per_cta = (long long)rp.h * g.wpl;
    ra.i = make_io(rp.in);
    ra.o = make_io(rp.out);
    ra.in_segs = rp.in_segs;
    ra.seg_len = rp.seg_len;
    ra.seg_stride = rp.seg_stride;
    const dim3 block(rp.threads);
    if (rp.tma) {
        TmaArgs ta{};
        ta.r = ra;
        ta.ntiles = (int)rp.ctas;
        ta.stages = rp.stages;
        ta.data_words = rp.h * rp.Ls;
        ta.sched_words = (int)ra.sched_words_per_cta;
        const dim3 grid((unsigned)rp.grid);
        const size_t smem = tma_smem(P, f);
        const bool cx = rp.out.cross != 0;
        const bool sg = rp.sg != 0;
        if (rp.split && rp.split_stg) {
            const bool dn = g.dense != 0;
            // the kernel derives its geometry from EPT (one line of 512 * EPT words per CTA)
            if ((int64_t(kStgWorkers) * rp.ept != (int64_t(1) << g.logL)) || g.E != 2 * g.logL - 5)
                return cudaErrorInvalidValue;
            CUtensorMap m{};
            if (map) m = *map;
            if (P.layout == 5 && P.tp[f].out_kind != 0) {
                // TLC ring pass: chunks of h1*h2 (X1) or h3*h2 (X2) words, one per block
                const long long h1 = P.tp[0].h, h2 = P.tp[1].h, h3 = P.tp[2].h;
                const int kind = P.tp[f].out_kind;
                const long long cw = kind == 1 ? h1 * h2 : h3 * h2;
                const long long nblk = kind == 1 ? P.c / h2 : P.r / h3;
                const long long bo = std::min<long long>(256, nblk / 2);
                ta.out_kind = kind;
                ta.chunk = (int)(cw / std::min<long long>(cw, 256));
                ta.box_outer = (int)bo;
                ta.box_words = (int)(bo * cw);
                ta.boxes_per_half = (int)(nblk / 2 / bo);
            }
            if (rp.ept == 32) return dn ? launch(row_pass_split_stg_kernel<32, true>, grid, block, smem, s, pdl, m, ta)
                                        : launch(row_pass_split_stg_kernel<32, false>, grid, block, smem, s, pdl, m, ta);
            if (rp.ept == 64) return dn ? launch(row_pass_split_stg_kernel<64, true>, grid, block, smem, s, pdl, m, ta)
                                        : launch(row_pass_split_stg_kernel<64, false>, grid, block, smem, s, pdl, m, ta);
            return cudaErrorInvalidValue;
        }
        if (rp.split) {
            const bool dn = g.dense != 0;
#define PERM_SPLIT_CASE(E_)                                                                               \
    case E_:                                                                                              \
        return dn ? launch(row_pass_split_kernel<E_, true, false>, grid, block, smem, s, pdl, ta)           \
                  : launch(row_pass_split_kernel<E_, false, false>, grid, block, smem, s, pdl, ta);
            switch (rp.ept) {
                PERM_SPLIT_CASE(8)
                PERM_SPLIT_CASE(16)
                PERM_SPLIT_CASE(32)
                PERM_SPLIT_CASE(64)
            }
#undef PERM_SPLIT_CASE
            return cudaErrorInvalidValue;
        }
#define PERM_TMA_CASE(E_)                                                                      \
    case E_:                                                                                   \
        if (sg) return cx ? launch(row_pass_tma_kernel<E_, true, true>, grid, block, smem, s, pdl, ta)  \
                          : launch(row_pass_tma_kernel<E_, false, true>, grid, block, smem, s, pdl, ta); \
        return cx ? launch(row_pass_tma_kernel<E_, true>, grid, block, smem, s, pdl, ta)       \
                  : launch(row_pass_tma_kernel<E_, false>, grid, block, smem, s, pdl, ta);
        switch (rp.ept) {
            PERM_TMA_CASE(4)
            PERM_TMA_CASE(8)
            PERM_TMA_CASE(16)
            PERM_TMA_CASE(32)
            PERM_TMA_CASE(64)
        }
#undef PERM_TMA_CASE
        return cudaErrorInvalidValue;
    }
    const dim3 grid((unsigned)rp.ctas);
    const size_t smem = row_smem(P, f);
    switch (rp.ept) {
        case 4: return launch(row_pass_kernel<4>, grid, block, smem, s, pdl, ra);
        case 8: return launch(row_pass_kernel<8>, grid, block, smem, s, pdl, ra);
        case 16: return launch(row_pass_kernel<16>, grid, block, smem, s, pdl, ra);
        case 32: return launch(row_pass_kernel<32>, grid, block, smem, s, pdl, ra);
        case 64: return launch(row_pass_kernel<64>, grid, block, smem, s, pdl, ra);
    }
    return cudaErrorInvalidValue;
}


cudaError_t launch_transpose(const uint32_t* in, uint32_t* out, int64_t rows, int64_t cols,
                             cudaStream_t s, bool pdl) {
    const dim3 grid((unsigned)(cols / 32), (unsigned)(rows / 32)), block(32, 8);
    if (rows >= 64 && cols >= 64)
        return launch(transpose64_kernel, dim3((unsigned)(cols / 64), (unsigned)(rows / 64)), dim3(256), 0,
                      s, pdl, in, out, ilog2i(rows), ilog2i(cols));
    return launch(transpose_kernel, grid, block, 0, s, pdl, in, out, ilog2i(rows), ilog2i(cols));
}

static unsigned stream_grid(long long nv) {
    long long want = (nv + 255) / 256;
    long long cap = (long long)sm_count() * 16;
    return (unsigned)(want < cap ? (want > 0 ? want : 1) : cap);
}

cudaError_t launch_scatter(const int32_t* p, const void* a, void* b, int64_t n, int eb,
                           cudaStream_t s) {
    const long long nv = n / 4;
    if (eb == 8)
        return launch(scatter64_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, p,
                      static_cast<const uint2*>(a), static_cast<uint2*>(b), nv);
    return launch(scatter_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, p,
                  static_cast<const uint32_t*>(a), static_cast<uint32_t*>(b), nv);
}

cudaError_t launch_gather(const int32_t* q, const void* a, void* b, int64_t n, int eb,
                          cudaStream_t s) {
    const long long nv = n / 4;
    if (eb == 8)
        return launch(gather64_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, q,
                      static_cast<const uint2*>(a), static_cast<uint2*>(b), nv);
    return launch(gather_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, q,
                  static_cast<const uint32_t*>(a), static_cast<uint32_t*>(b), nv);
}

cudaError_t launch_block_gather(const int32_t* qb, const void* a, void* b, int64_t n_words,
                                cudaStream_t s) {
    const long long nv = n_words / 4;
    return launch(block_gather_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, qb,
                  static_cast<const uint32_t*>(a), static_cast<uint32_t*>(b), nv);
}

cudaError_t launch_copy(const uint32_t* a, uint32_t* b, int64_t n, cudaStream_t s) {
    const long long nv = n / 4;
    return launch(copy_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, a, b, nv);
}

}  // namespace perm
