// gplan.cu — the offline colourings of the plan builder on the GPU.
//
// PAPER.md Thm 6 (L515) only proves that a d-regular bipartite multigraph has a
// proper d-edge-colouring (König); the paper colours offline and never times it.
// Both colourings of the method are of that kind and every degree here is a
// power of two, so we use Euler splitting, as the host planner does
// (planner.cpp), restructured for thousands of threads:
//
//   level l (degree d = d0 >> l, edges grouped in aligned blocks of d per
//   vertex on each side, ordU / ordV = edge ids in block order):
//   1. pair positions (2i, 2i+1) of every block: partner_U(e), partner_V(e);
//   2. the pairings form disjoint cycles alternating V- and U-links; the map
//      g = partner_U o partner_V walks every second edge of a cycle, so each
//      cycle is two g-orbits and colouring one orbit 0 and the other 1 gives
//      every vertex exactly half its edges of each colour;
//   3. orbit labels by a ruling set: ~1/32 of the edges (hash-selected) are
//      rulers; each ruler walks g to the next ruler and stamps its segment; the
//      rulers (plus the edges of ruler-free orbits, which are short) then find
//      the minimum ruler id of their orbit by synchronous pointer jumping over
//      a compacted list: O(E) work per level instead of O(E log E);
//   4. colour bit b(e) = [label(e) < label(partner_V(e))] (the two orbits of a
//      cycle have different labels);
//   5. stable split of every block into its b = 0 half and its b = 1 half
//      (a pair holds one edge of each colour, so the destination of position
//      2i + j is block*d + b*d/2 + i: no scan).
//   After log2(d0) levels every block is one edge: colour(ordU[q]) = q mod d0.
//
// Row level (a1): vertices = source rows (edge x in block x >> log c, i.e.
// ordU = identity) and destination rows (ordV[P(x)] = x), d0 = c.
// Bank level (a3, per line or per TLC tile of B elements): vertices =
// (block, source bank) and (block, destination bank), d0 = B / 32.
// The result is checked like the host planner's: by the oracle's invariants.

#include <cuda_runtime.h>

#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "gplan.hpp"

namespace perm {

namespace {

constexpr int kRulerLog = 5;   // 1 in 32 edges starts a walk

__device__ __forceinline__ uint32_t mix32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352du;
    x ^= x >> 15; x *= 0x846ca68bu;
    x ^= x >> 16;
    return x;
}
__device__ __forceinline__ bool is_ruler(uint32_t e, uint32_t seed) {
    return (mix32(e ^ seed) & ((1u << kRulerLog) - 1u)) == 0u;
}

__global__ void k_pair(const uint32_t* __restrict__ ord, uint32_t* __restrict__ partner, int64_t E) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < E; q += (int64_t)gridDim.x * blockDim.x)
        partner[ord[q]] = ord[q ^ 1];
}

__global__ void k_compose(const uint32_t* __restrict__ pU, const uint32_t* __restrict__ pV,
                          uint32_t* __restrict__ g, int64_t E) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x)
        g[e] = pU[pV[e]];
}

// every ruler stamps its segment (itself and the non-rulers up to the next ruler)
__global__ void k_walk(const uint32_t* __restrict__ g, uint32_t* __restrict__ seg,
                       uint32_t* __restrict__ nxt, int64_t E, uint32_t seed) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
        if (!is_ruler((uint32_t)e, seed)) continue;
        seg[e] = (uint32_t)e;
        uint32_t x = g[e];
        while (!is_ruler(x, seed)) {
            seg[x] = (uint32_t)e;
            x = g[x];
        }
        nxt[e] = x;
    }
}

// nodes of the reduced graph: rulers (next = next ruler) and the edges of
// ruler-free orbits (seg still ~0: next = g); compacted into list slots
__global__ void k_compact(const uint32_t* __restrict__ g, uint32_t* __restrict__ seg,
                          uint32_t* __restrict__ nxt, uint32_t* __restrict__ slotof,
                          uint32_t* __restrict__ node, unsigned long long* __restrict__ count, int64_t E) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
        uint32_t s = seg[e];
        if (s == 0xFFFFFFFFu) {
            seg[e] = (uint32_t)e;
            nxt[e] = g[e];
            s = (uint32_t)e;
        }
        // warp-aggregated slot allocation: one atomic per warp (for short-orbit inputs,
        // e.g. identity, nearly every edge is a node)
        const bool is_node = s == (uint32_t)e;
        const unsigned act = __activemask();
        const unsigned bal = __ballot_sync(act, is_node);
        const int leader = __ffs(act) - 1, lane = threadIdx.x & 31;
        unsigned long long base = 0;
        if (lane == leader && bal) base = atomicAdd(count, (unsigned long long)__popc(bal));
        base = __shfl_sync(act, base, leader);
        if (is_node) {
            const uint32_t slot = (uint32_t)(base + __popc(bal & ((1u << lane) - 1u)));
            slotof[e] = slot;
            node[slot] = (uint32_t)e;
        }
    }
}

__global__ void k_reduced_init(const uint32_t* __restrict__ node, const uint32_t* __restrict__ nxt,
                               const uint32_t* __restrict__ slotof, uint32_t* __restrict__ lab,
                               uint32_t* __restrict__ nx, int64_t R) {
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < R; s += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t e = node[s];
        lab[s] = e;
        nx[s] = slotof[nxt[e]];
    }
}

// synchronous pointer jumping (ping-pong buffers): after round j, lab = min over
// the next 2^j nodes of the orbit; a round without a change means converged
__global__ void k_jump(const uint32_t* __restrict__ lab, const uint32_t* __restrict__ nx,
                       uint32_t* __restrict__ lab2, uint32_t* __restrict__ nx2, int64_t R,
                       int* __restrict__ changed) {
    int ch = 0;
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < R; s += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t n1 = nx[s];
        const uint32_t a = lab[s], b = lab[n1];
        const uint32_t m = b < a ? b : a;
        ch |= m != a;
        lab2[s] = m;
        nx2[s] = nx[n1];
    }
    if (__syncthreads_or(ch) && threadIdx.x == 0) *changed = 1;
}

__global__ void k_label(const uint32_t* __restrict__ seg, const uint32_t* __restrict__ slotof,
                        const uint32_t* __restrict__ rlab, uint32_t* __restrict__ lab, int64_t E) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x)
        lab[e] = rlab[slotof[seg[e]]];
}

// colour bit of every edge: b(e) = [label(e) >= label(partner_V(e))]
__global__ void k_bit(const uint32_t* __restrict__ lab, const uint32_t* __restrict__ pV,
                      uint8_t* __restrict__ bit, int64_t E) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x)
        bit[e] = lab[e] < lab[pV[e]] ? 0 : 1;
}

__global__ void k_split(const uint32_t* __restrict__ ord, uint32_t* __restrict__ ord2,
                        const uint8_t* __restrict__ bit, int64_t E, int logd) {
    const int64_t half = (int64_t)1 << (logd - 1);
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < E; q += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t e = ord[q];
        const int64_t blk = q >> logd, i = (q & ((half << 1) - 1)) >> 1;
        ord2[(blk << logd) + (int64_t)bit[e] * half + i] = e;
    }
}

__global__ void k_final(const uint32_t* __restrict__ ord, uint16_t* __restrict__ col, int64_t E, uint32_t dmask) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < E; q += (int64_t)gridDim.x * blockDim.x)
        col[ord[q]] = (uint16_t)(q & dmask);
}

__global__ void k_row_orders(const int32_t* __restrict__ p, uint32_t* __restrict__ ordU,
                             uint32_t* __restrict__ ordV, int64_t n) {
    for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n; x += (int64_t)gridDim.x * blockDim.x) {
        ordU[x] = (uint32_t)x;
        ordV[p[x]] = (uint32_t)x;      // sorted by P(x): blocks of c per destination row
    }
}

// bank level: block of B = 2^logB elements (a line or a TLC tile); vertex
// (block, key & 31) on each side, position (key & 31) * B/32 + (key >> 5)
__global__ void k_bank_orders(const uint16_t* __restrict__ keyU, const uint16_t* __restrict__ keyV,
                              uint32_t* __restrict__ ordU, uint32_t* __restrict__ ordV, int64_t E, int logB) {
    const int sh = logB - 5;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t base = (e >> logB) << logB;
        const uint32_t ku = keyU ? (uint32_t)keyU[e] : (uint32_t)(e & ((1 << logB) - 1)), kv = keyV[e];
        ordU[base + ((int64_t)(ku & 31) << sh) + (ku >> 5)] = (uint32_t)e;
        ordV[base + ((int64_t)(kv & 31) << sh) + (kv >> 5)] = (uint32_t)e;
    }
}

using gclk = std::chrono::steady_clock;
double gms(gclk::time_point t0) { return std::chrono::duration<double, std::milli>(gclk::now() - t0).count(); }
bool gverbose() {
    static const bool v = std::getenv("PERM_PLANNER_VERBOSE") != nullptr;
    return v;
}

// W64 packing (plan.hpp entry_pos): element e = (line, j) with bank colour col[e]
// sits at slot q = col*32 + (j mod 32) of its line; entry (sigma << logL) | t
__global__ void k_w64_entries(const uint16_t* __restrict__ phi, const uint16_t* __restrict__ col,
                              uint32_t* __restrict__ ent, int64_t n, int logL) {
    const int64_t Lm = ((int64_t)1 << logL) - 1;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = e & Lm;
        const int64_t q = (int64_t)col[e] * 32 + (j & 31);
        ent[(e & ~Lm) + q] = ((uint32_t)(j >> 5) << logL) | phi[e];
    }
}
// 64-bit word w = (line*(L/32) + round)*w64 + wsel holds lanes wsel*epw .. of the round
__global__ void k_w64_pack(const uint32_t* __restrict__ ent, uint32_t* __restrict__ words, int64_t nw64,
                           int E, int epw, int w64) {
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nw64; w += (int64_t)gridDim.x * blockDim.x) {
        const int64_t lr = w / w64;
        const int wsel = (int)(w - lr * w64);
        const uint32_t* src = ent + lr * 32;
        uint64_t v = 0;
        for (int i = 0; i < epw; ++i) {
            const int x = wsel * epw + i;
            if (x < 32) v |= (uint64_t)src[x] << (E * i);
        }
        words[2 * w] = (uint32_t)v;
        words[2 * w + 1] = (uint32_t)(v >> 32);
    }
}

// dense format: round lr = E u32 words, lane x's entry at bit x*E; thread per word
__global__ void k_dense_pack(const uint32_t* __restrict__ ent, uint32_t* __restrict__ words, int64_t nwords,
                             int E) {
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nwords; w += (int64_t)gridDim.x * blockDim.x) {
        const int64_t lr = w / E;
        const int wi = (int)(w - lr * E);
        const uint32_t* src = ent + lr * 32;
        const int x0 = (32 * wi) / E, x1 = min(31, (32 * wi + 31) / E);
        uint32_t v = 0;
        for (int x = x0; x <= x1; ++x) {
            const int pos = x * E - 32 * wi;
            const uint64_t e = src[x];
            v |= pos >= 0 ? (uint32_t)(e << pos) : (uint32_t)(e >> -pos);
        }
        words[w] = v;
    }
}

struct DevBuf {
    void* p = nullptr;
    ~DevBuf() { if (p) cudaFree(p); }
};

#define GP_TRY(x)                              \
    do {                                       \
        cudaError_t e_ = (x);                  \
        if (e_ != cudaSuccess) return e_;      \
    } while (0)

unsigned grid_for(int64_t E) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t want = (E + 255) / 256;
    const int64_t cap = (int64_t)sms * 8;
    return (unsigned)(want < cap ? (want > 0 ? want : 1) : cap);
}

// Euler split of the blocks in ordU / ordV (device, E edges, degree 2^logd0);
// writes colour[e] in [0, 2^logd0). ordU / ordV are clobbered.
cudaError_t euler_split_device(uint32_t* ordU, uint32_t* ordV, int64_t E, int logd0, uint16_t* colour,
                               cudaStream_t s, GpuPlanStats* st) {
    const unsigned G = grid_for(E), T = 256;
    const bool verbose = gverbose();
    auto ta = gclk::now();
    DevBuf bU2, bV2, bpU, bpV, bg, bseg, bnxt, bslot, bnode, blab, blab2, bnx, bnx2, bcnt, bch;
    const size_t W = (size_t)E * 4;
    GP_TRY(cudaMalloc(&bU2.p, W));
    GP_TRY(cudaMalloc(&bV2.p, W));
    GP_TRY(cudaMalloc(&bpU.p, W));
    GP_TRY(cudaMalloc(&bpV.p, W));
    GP_TRY(cudaMalloc(&bg.p, W));
    GP_TRY(cudaMalloc(&bseg.p, W));
    GP_TRY(cudaMalloc(&bnxt.p, W));
    GP_TRY(cudaMalloc(&bslot.p, W));
    GP_TRY(cudaMalloc(&bnode.p, W));
    GP_TRY(cudaMalloc(&blab.p, W));
    GP_TRY(cudaMalloc(&blab2.p, W));
    GP_TRY(cudaMalloc(&bnx.p, W));
    GP_TRY(cudaMalloc(&bnx2.p, W));
    GP_TRY(cudaMalloc(&bcnt.p, 8));
    GP_TRY(cudaMalloc(&bch.p, 4));
    uint32_t *U = ordU, *V = ordV, *U2 = (uint32_t*)bU2.p, *V2 = (uint32_t*)bV2.p;
    uint32_t *pU = (uint32_t*)bpU.p, *pV = (uint32_t*)bpV.p, *g = (uint32_t*)bg.p;
    uint32_t *seg = (uint32_t*)bseg.p, *nxt = (uint32_t*)bnxt.p, *slotof = (uint32_t*)bslot.p;
    uint32_t *node = (uint32_t*)bnode.p, *lab = (uint32_t*)blab.p, *lab2 = (uint32_t*)blab2.p;
    uint32_t *nx = (uint32_t*)bnx.p, *nx2 = (uint32_t*)bnx2.p;
    unsigned long long* cnt = (unsigned long long*)bcnt.p;
    int* changed = (int*)bch.p;
    if (verbose) {
        cudaStreamSynchronize(s);
        std::fprintf(stderr, "[gplan] E=%lld logd0=%d alloc %.1f ms\n", (long long)E, logd0, gms(ta));
    }
    for (int l = 0; l < logd0; ++l) {
        const int logd = logd0 - l;
        auto tl = gclk::now();
        int rounds = 0;
        k_pair<<<G, T, 0, s>>>(U, pU, E);
        k_pair<<<G, T, 0, s>>>(V, pV, E);
        k_compose<<<G, T, 0, s>>>(pU, pV, g, E);
        GP_TRY(cudaMemsetAsync(seg, 0xFF, W, s));
        GP_TRY(cudaMemsetAsync(cnt, 0, 8, s));
        const uint32_t seed = 0x9E3779B9u * (uint32_t)(l + 1);
        k_walk<<<G, T, 0, s>>>(g, seg, nxt, E, seed);
        k_compact<<<G, T, 0, s>>>(g, seg, nxt, slotof, node, cnt, E);
        unsigned long long R = 0;
        GP_TRY(cudaMemcpyAsync(&R, cnt, 8, cudaMemcpyDeviceToHost, s));
        GP_TRY(cudaStreamSynchronize(s));
        const unsigned GR = grid_for((int64_t)R);
        k_reduced_init<<<GR, T, 0, s>>>(node, nxt, slotof, lab, nx, (int64_t)R);
        uint32_t *la = lab, *lb = lab2, *na = nx, *nb = nx2;
        for (int round = 0;; ++round) {
            int h = 0;
            GP_TRY(cudaMemsetAsync(changed, 0, 4, s));
            k_jump<<<GR, T, 0, s>>>(la, na, lb, nb, (int64_t)R, changed);
            GP_TRY(cudaMemcpyAsync(&h, changed, 4, cudaMemcpyDeviceToHost, s));
            GP_TRY(cudaStreamSynchronize(s));
            std::swap(la, lb);
            std::swap(na, nb);
            if (st) st->jump_rounds += 1;
            ++rounds;
            if (!h || round > 64) break;
        }
        // la = final labels of the reduced nodes; spread to every edge (into lb: free)
        k_label<<<G, T, 0, s>>>(seg, slotof, la, lb, E);
        uint8_t* bit = reinterpret_cast<uint8_t*>(g);      // g is dead after the walk
        k_bit<<<G, T, 0, s>>>(lb, pV, bit, E);
        k_split<<<G, T, 0, s>>>(U, U2, bit, E, logd);
        k_split<<<G, T, 0, s>>>(V, V2, bit, E, logd);
        std::swap(U, U2);
        std::swap(V, V2);
        if (st) { st->levels += 1; st->reduced_nodes += (int64_t)R; }
        GP_TRY(cudaGetLastError());
        if (verbose) {
            cudaStreamSynchronize(s);
            std::fprintf(stderr, "[gplan]  level %d: reduced %llu, %d jump rounds, %.2f ms\n", l,
                         (unsigned long long)R, rounds, gms(tl));
        }
    }
    k_final<<<G, T, 0, s>>>(U, colour, E, (uint32_t)((1u << logd0) - 1u));
    GP_TRY(cudaGetLastError());
    return cudaStreamSynchronize(s);
}

}  // namespace

cudaError_t gpu_row_colour(const int32_t* p_host, int64_t n, int logc, uint16_t* kappa_host,
                           GpuPlanStats* st) {
    auto t0 = gclk::now();
    cudaStream_t s = nullptr;
    GP_TRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
    DevBuf bp, bU, bV, bc;
    GP_TRY(cudaMalloc(&bp.p, (size_t)n * 4));
    GP_TRY(cudaMalloc(&bU.p, (size_t)n * 4));
    GP_TRY(cudaMalloc(&bV.p, (size_t)n * 4));
    GP_TRY(cudaMalloc(&bc.p, (size_t)n * 2));
    GP_TRY(cudaMemcpyAsync(bp.p, p_host, (size_t)n * 4, cudaMemcpyHostToDevice, s));
    k_row_orders<<<grid_for(n), 256, 0, s>>>((const int32_t*)bp.p, (uint32_t*)bU.p, (uint32_t*)bV.p, n);
    GP_TRY(cudaGetLastError());
    cudaFree(bp.p);
    bp.p = nullptr;
    if (gverbose()) {
        cudaStreamSynchronize(s);
        std::fprintf(stderr, "[gplan] row colour: alloc + upload p + orders %.1f ms\n", gms(t0));
    }
    GP_TRY(euler_split_device((uint32_t*)bU.p, (uint32_t*)bV.p, n, logc, (uint16_t*)bc.p, s, st));
    auto t1 = gclk::now();
    GP_TRY(cudaMemcpyAsync(kappa_host, bc.p, (size_t)n * 2, cudaMemcpyDeviceToHost, s));
    const cudaError_t e = cudaStreamSynchronize(s);
    if (gverbose()) std::fprintf(stderr, "[gplan] row colour: download %.1f ms, total %.1f ms\n", gms(t1), gms(t0));
    return e;
}

cudaError_t gpu_bank_colour(const uint16_t* keyU_host, const uint16_t* keyV_host, int64_t E, int logB,
                            uint16_t* col_host, GpuPlanStats* st) {
    // B = 32 (a 32-element line): degree 1, every edge gets colour 0 (no split level)
    if (logB < 5 || logB > 16 || (E & ((int64_t(1) << logB) - 1))) return cudaErrorInvalidValue;
    auto t0 = gclk::now();
    cudaStream_t s = nullptr;
    GP_TRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
    DevBuf bku, bkv, bU, bV, bc;
    if (keyU_host) GP_TRY(cudaMalloc(&bku.p, (size_t)E * 2));
    GP_TRY(cudaMalloc(&bkv.p, (size_t)E * 2));
    GP_TRY(cudaMalloc(&bU.p, (size_t)E * 4));
    GP_TRY(cudaMalloc(&bV.p, (size_t)E * 4));
    GP_TRY(cudaMalloc(&bc.p, (size_t)E * 2));
    if (keyU_host) GP_TRY(cudaMemcpyAsync(bku.p, keyU_host, (size_t)E * 2, cudaMemcpyHostToDevice, s));
    GP_TRY(cudaMemcpyAsync(bkv.p, keyV_host, (size_t)E * 2, cudaMemcpyHostToDevice, s));
    k_bank_orders<<<grid_for(E), 256, 0, s>>>((const uint16_t*)bku.p, (const uint16_t*)bkv.p,
                                              (uint32_t*)bU.p, (uint32_t*)bV.p, E, logB);
    GP_TRY(cudaGetLastError());
    if (gverbose()) {
        cudaStreamSynchronize(s);
        std::fprintf(stderr, "[gplan] bank colour: alloc + upload keys + orders %.1f ms\n", gms(t0));
    }
    GP_TRY(euler_split_device((uint32_t*)bU.p, (uint32_t*)bV.p, E, logB - 5, (uint16_t*)bc.p, s, st));
    auto t1 = gclk::now();
    GP_TRY(cudaMemcpyAsync(col_host, bc.p, (size_t)E * 2, cudaMemcpyDeviceToHost, s));
    const cudaError_t e = cudaStreamSynchronize(s);
    if (gverbose()) std::fprintf(stderr, "[gplan] bank colour: download %.1f ms, total %.1f ms\n", gms(t1), gms(t0));
    return e;
}

}  // namespace perm

namespace perm {

cudaError_t gpu_line_schedules(const uint16_t* phi_host, int64_t n, int logL, int E, int epw, int w64,
                               int dense, uint32_t* words_host, GpuPlanStats* st) {
    if (logL < 5 || logL > 16 || (n & ((int64_t(1) << logL) - 1))) return cudaErrorInvalidValue;
    auto t0 = gclk::now();
    cudaStream_t s = nullptr;
    GP_TRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    struct SG { cudaStream_t s; ~SG() { cudaStreamDestroy(s); } } sg{s};
    DevBuf bph, bU, bV, bc;
    GP_TRY(cudaMalloc(&bph.p, (size_t)n * 2));
    GP_TRY(cudaMalloc(&bU.p, (size_t)n * 4));
    GP_TRY(cudaMalloc(&bV.p, (size_t)n * 4));
    GP_TRY(cudaMalloc(&bc.p, (size_t)n * 2));
    GP_TRY(cudaMemcpyAsync(bph.p, phi_host, (size_t)n * 2, cudaMemcpyHostToDevice, s));
    k_bank_orders<<<grid_for(n), 256, 0, s>>>(nullptr, (const uint16_t*)bph.p, (uint32_t*)bU.p, (uint32_t*)bV.p,
                                              n, logL);
    GP_TRY(cudaGetLastError());
    GP_TRY(euler_split_device((uint32_t*)bU.p, (uint32_t*)bV.p, n, logL - 5, (uint16_t*)bc.p, s, st));
    // ordU / ordV are free now: entries into U, packed words into V (W64 words <= n)
    const int64_t nw64 = (n / 32) * w64;
    const int64_t nw32 = dense ? (n / 32) * E : 2 * nw64;     // <= n u32 either way
    k_w64_entries<<<grid_for(n), 256, 0, s>>>((const uint16_t*)bph.p, (const uint16_t*)bc.p, (uint32_t*)bU.p, n,
                                              logL);
    if (dense)
        k_dense_pack<<<grid_for(nw32), 256, 0, s>>>((const uint32_t*)bU.p, (uint32_t*)bV.p, nw32, E);
    else
        k_w64_pack<<<grid_for(nw64), 256, 0, s>>>((const uint32_t*)bU.p, (uint32_t*)bV.p, nw64, E, epw, w64);
    GP_TRY(cudaGetLastError());
    auto t1 = gclk::now();
    GP_TRY(cudaMemcpyAsync(words_host, bV.p, (size_t)nw32 * 4, cudaMemcpyDeviceToHost, s));
    const cudaError_t e = cudaStreamSynchronize(s);
    if (gverbose())
        std::fprintf(stderr, "[gplan] line schedules: download %.1f ms, total %.1f ms\n", gms(t1), gms(t0));
    return e;
}

}  // namespace perm
