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
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.hpp"

namespace perm {

namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;

__device__ __forceinline__ void pdl_wait() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
}
__device__ __forceinline__ void pdl_launch_dependents() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void prefetch_l2(const void* p) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
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

// Entry of this lane from the E words of one warp-round held one per lane
// (lane j holds word j): bits [E*lane, E*lane + E).
__device__ __forceinline__ uint32_t decode_entry(uint32_t word, int w0, int off, uint32_t mask) {
    const uint32_t lo = __shfl_sync(kFull, word, w0);
    const uint32_t hi = __shfl_sync(kFull, word, w0 + 1);
    return __funnelshift_r(lo, hi, off) & mask;
}

// ------------------------------------------------------------------ permute hop

// In-place permutation of the lines resident in shared memory. Warp-round q
// (0 <= q < h*L/32) of this CTA is line q >> (logL-5), round q & (L/32 - 1);
// warp w handles q = w + W*m for m < EPT. addr(l, pos) maps (line, position)
// to a shared-memory word: ROWS -> l*Ls + pos, COLS -> pos*Ls + l.
template <int EPT, bool COLS>
__device__ __forceinline__ void permute_lines(uint32_t* sm, const uint32_t* __restrict__ sched,
                                              int logL, int E, int Ls) {
    const int tid = threadIdx.x, lane = tid & 31, W = blockDim.x >> 5;
    const int logR = logL - 5;                      // log2(rounds per line)
    const int bit0 = E * lane, w0 = bit0 >> 5, off = bit0 & 31;
    const uint32_t mask = (1u << E) - 1u;
    const uint32_t tmask = (1u << logL) - 1u;
    const bool has_word = lane < E;
    const int WE = W * E;
    constexpr int CH = EPT < 8 ? EPT : 8;
    uint32_t v[EPT];
    // read hop: v[m] = line[32*sigma + lane]   (bank = lane + const: conflict-free)
    {
        const int warp = tid >> 5;
        const uint32_t* sp = sched + warp * E + lane;
#pragma unroll
        for (int c0 = 0; c0 < EPT; c0 += CH) {
            uint32_t sw[CH];
#pragma unroll
            for (int u = 0; u < CH; ++u) sw[u] = has_word ? __ldg(sp + (c0 + u) * WE) : 0u;
#pragma unroll
            for (int u = 0; u < CH; ++u) {
                const int l = (warp + W * (c0 + u)) >> logR;
                const uint32_t e = decode_entry(sw[u], w0, off, mask);
                const int s = (int)((e >> logL) << 5) + lane;
                v[c0 + u] = COLS ? sm[s * Ls + l] : sm[l * Ls + s];
            }
        }
    }
    __syncthreads();
    // write hop: line[t] = v[m]   (the 32 t of a warp-round hit 32 distinct banks).
    // The warp index is re-read through a shuffle so the compiler recomputes the
    // per-round addresses instead of keeping EPT of them live across the barrier.
    {
        const int warp = __shfl_sync(kFull, tid >> 5, 0);
        const uint32_t* sp = sched + warp * E + lane;
#pragma unroll
        for (int c0 = 0; c0 < EPT; c0 += CH) {
            uint32_t sw[CH];
#pragma unroll
            for (int u = 0; u < CH; ++u) sw[u] = has_word ? __ldg(sp + (c0 + u) * WE) : 0u;
#pragma unroll
            for (int u = 0; u < CH; ++u) {
                const int l = (warp + W * (c0 + u)) >> logR;
                const uint32_t e = decode_entry(sw[u], w0, off, mask);
                const int t = (int)(e & tmask);
                if (COLS) sm[t * Ls + l] = v[c0 + u];
                else      sm[l * Ls + t] = v[c0 + u];
            }
        }
    }
    __syncthreads();
}

// ------------------------------------------------------------------ fused (n <= 2^15)

struct FusedArgs {
    const uint32_t* in;
    uint32_t* out;
    const uint32_t* sched[3];
    int logr, logc, Ls, E[3];
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
    permute_lines<EPT, false>(sm, a.sched[0], a.logc, a.E[0], a.Ls);   // Step 1: rows
    permute_lines<EPT, true>(sm, a.sched[1], a.logr, a.E[1], a.Ls);    // Step 2: columns
    permute_lines<EPT, false>(sm, a.sched[2], a.logc, a.E[2], a.Ls);   // Step 3: rows
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
    int logL, logh, Ls, E;
    long long sched_words_per_cta;
    Io i, o;
};

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
    if (!m.cross) {
        const int loghw = a.logh + m.logw;
#pragma unroll
        for (int it = 0; it < NV; ++it) {
            const int f = 4 * (tid + T * it);
            const int K = f >> loghw, rem = f & ((1 << loghw) - 1);
            val[it] = ld_nc_v4(base + (long long)K * m.strideK + rem);
        }
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
__global__ void __launch_bounds__(512, 1) row_pass_kernel(const RowArgs a) {
    extern __shared__ __align__(16) uint32_t sm[];
    const long long cta = blockIdx.x;
    const uint32_t* sched = a.sched + cta * a.sched_words_per_cta;
    // The schedule does not depend on the previous pass: pull it into L2 while
    // the previous kernel drains (32 words = one 128-byte line per thread step).
    for (long long w = (long long)threadIdx.x * 32; w < a.sched_words_per_cta;
         w += (long long)blockDim.x * 32)
        prefetch_l2(sched + w);
    pdl_wait();
    tile_load<EPT>(a, sm, cta);
    __syncthreads();
    pdl_launch_dependents();
    permute_lines<EPT, false>(sm, sched, a.logL, a.E, a.Ls);
    tile_store<EPT>(a, sm, cta);
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

}  // namespace

cudaError_t prepare_kernels(const HostPlan& P) {
    cudaError_t e = cudaSuccess;
    auto set = [&](const void* k, size_t bytes) {
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    };
    if (P.passes == 1) {
        const size_t b = fused_smem(P);
        switch (P.fused_ept) {
            case 4: set((const void*)fused_kernel<4>, b); break;
            case 8: set((const void*)fused_kernel<8>, b); break;
            case 16: set((const void*)fused_kernel<16>, b); break;
            case 32: set((const void*)fused_kernel<32>, b); break;
            case 64: set((const void*)fused_kernel<64>, b); break;
            default: return cudaErrorInvalidValue;
        }
        return e;
    }
    // one attribute per template instance: use the largest request among the passes
    size_t need[7] = {0, 0, 0, 0, 0, 0, 0};   // index log2(ept)
    for (int f = 0; f < 3; ++f) {
        const int li = ilog2i(P.rp[f].ept);
        if (li < 2 || li > 6) return cudaErrorInvalidValue;
        need[li] = need[li] > row_smem(P, f) ? need[li] : row_smem(P, f);
    }
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
        case 64: return launch(fused_kernel<64>, grid, block, smem, s, false, fa);
    }
    return cudaErrorInvalidValue;
}

cudaError_t launch_row_pass(const HostPlan& P, int f, const uint32_t* sched, const uint32_t* in,
                            uint32_t* out, cudaStream_t s, bool pdl) {
    const RowPass& rp = P.rp[f];
    const PhaseGeom& g = P.ph[rp.phase];
    RowArgs ra{};
    ra.in = in;
    ra.out = out;
    ra.sched = sched;
    ra.logL = g.logL;
    ra.logh = ilog2i(rp.h);
    ra.Ls = rp.Ls;
    ra.E = g.E;
    ra.sched_words_per_cta = (long long)rp.h * (g.L / 32) * g.E;
    ra.i = make_io(rp.in);
    ra.o = make_io(rp.out);
    const dim3 grid((unsigned)rp.ctas), block(rp.threads);
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
    return launch(transpose_kernel, grid, block, 0, s, pdl, in, out, ilog2i(rows), ilog2i(cols));
}

static unsigned stream_grid(long long nv) {
    long long want = (nv + 255) / 256;
    long long cap = (long long)sm_count() * 16;
    return (unsigned)(want < cap ? (want > 0 ? want : 1) : cap);
}

cudaError_t launch_scatter(const int32_t* p, const uint32_t* a, uint32_t* b, int64_t n,
                           cudaStream_t s) {
    const long long nv = n / 4;
    return launch(scatter_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, p, a, b, nv);
}

cudaError_t launch_gather(const int32_t* q, const uint32_t* a, uint32_t* b, int64_t n,
                          cudaStream_t s) {
    const long long nv = n / 4;
    return launch(gather_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, q, a, b, nv);
}

cudaError_t launch_copy(const uint32_t* a, uint32_t* b, int64_t n, cudaStream_t s) {
    const long long nv = n / 4;
    return launch(copy_kernel, dim3(stream_grid(nv)), dim3(256), 0, s, false, a, b, nv);
}

}  // namespace perm
