// planner.cpp — offline plan builder of libperm (host, C++17 + OpenMP).
//
// PAPER.md §VII (L603-L605, L537-L539) and §VI (L515-L533):
//  1. validate P (L361: p holds a permutation of 0..n-1);
//  2. view the arrays as r x c (L603, "not restricted to a square matrix");
//  3. colour the c-regular row-level bipartite multigraph (U = source rows,
//     V = destination rows, one edge per element) with c colours (Thm 6);
//  4. derive the three per-line permutations Phi1 (colour k -> column k),
//     Phi2 (within column k, to the destination row), Phi3 (within the
//     destination row, to the destination column);
//  5. for every line of every phase colour its (L/32)-regular bank-level
//     graph (edge (j mod 32, Phi(j) mod 32)) with L/32 colours: colour k is
//     warp-round k, and lane x takes the colour-k edge leaving bank x
//     (s = 32*sigma + x, t = Phi(s));
//  6. pack (sigma, t) into 2*log2(L)-5 bit entries.
//
// The paper proves the colourings exist (König) but gives no algorithm; we
// use Euler splitting, valid because every degree here is a power of two:
// pair the edges at every node, the pairings form disjoint even alternating
// cycles, colour each cycle 0,1,0,1,...: every node keeps exactly half its
// edges on each side. Recurse log2(d) times. O(E log d).
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <new>
#include <numeric>
#include <utility>

#ifdef _OPENMP
#include <omp.h>
#endif

#include "plan.hpp"
#include "gplan.hpp"

namespace perm {

namespace {

using clk = std::chrono::steady_clock;
double ms_since(clk::time_point t0) {
    return std::chrono::duration<double, std::milli>(clk::now() - t0).count();
}

int ilog2(int64_t v) {
    int k = 0;
    while ((int64_t(1) << k) < v) ++k;
    return k;
}

int64_t pow2_floor(int64_t v) {
    if (v < 1) return 1;
    int64_t p = 1;
    while (p * 2 <= v) p *= 2;
    return p;
}

constexpr uint32_t kNone = 0xFFFFFFFFu;

// Reusable Euler-split colourer (scratch kept across calls).
struct EulerColourer {
    std::vector<uint32_t> ord, ord2, pu, pu2, pv, pv2, pL, pR;
    std::vector<uint8_t> bit;

    void split_group(int64_t base, int64_t S, int64_t nodes, std::vector<uint32_t>& pend) {
        // pair consecutive incident edges at every left node, then every right node
        std::fill(pend.begin(), pend.begin() + nodes, kNone);
        for (int64_t i = base; i < base + S; ++i) {
            uint32_t& q = pend[pu[i]];
            if (q == kNone) q = (uint32_t)i;
            else { pL[i] = q; pL[q] = (uint32_t)i; q = kNone; }
        }
        std::fill(pend.begin(), pend.begin() + nodes, kNone);
        for (int64_t i = base; i < base + S; ++i) {
            uint32_t& q = pend[pv[i]];
            if (q == kNone) q = (uint32_t)i;
            else { pR[i] = q; pR[q] = (uint32_t)i; q = kNone; }
        }
        // walk the alternating cycles, colouring 0,1,0,1,...
        std::memset(bit.data() + base, 2, (size_t)S);
        for (int64_t i = base; i < base + S; ++i) {
            if (bit[i] != 2) continue;
            uint32_t cur = (uint32_t)i;
            do {
                bit[cur] = 0;
                uint32_t nx = pL[cur];
                bit[nx] = 1;
                cur = pR[nx];
            } while (cur != (uint32_t)i);
        }
        // stable partition: bit 0 first half, bit 1 second half
        int64_t z = base, o = base + S / 2;
        for (int64_t i = base; i < base + S; ++i) {
            int64_t dst = bit[i] ? o++ : z++;
            ord2[dst] = ord[i];
            pu2[dst] = pu[i];
            pv2[dst] = pv[i];
        }
    }

    // The same split of one big group by all threads (top recursion levels, where
    // there are fewer groups than threads). (1) pairing: every thread pairs the edges
    // of its chunk at each node; the at most one leftover per node per thread is
    // paired sequentially. (2) the alternating cycles are coloured by concurrent
    // walks: a walk claims edges (CAS on owner[]) in both directions from its start
    // and stops at the first edge another walk owns, recording that boundary; every
    // walk is a segment with tentative bits. (3) the boundaries give parity
    // constraints between segments (bits of adjacent edges must differ), solved by
    // BFS; (4) flipped segments' bits are inverted; (5) parallel stable partition.
    std::vector<int32_t> owner;

    void split_group_par(int64_t base, int64_t S, int64_t nodes) {
        static const bool verbose = std::getenv("PERM_PLANNER_VERBOSE") != nullptr;
        auto t0 = clk::now();
#ifdef _OPENMP
        const int T = omp_get_max_threads();
#else
        const int T = 1;
#endif
        // a fixed chunking (not the thread count) keeps the pairing, and so the colouring,
        // identical on every rank / machine: sharded plans rely on it
        constexpr int NCH = 64;
        std::vector<std::vector<uint32_t>> leftL(NCH), leftR(NCH);
#pragma omp parallel for schedule(dynamic, 1)
        for (int ch = 0; ch < NCH; ++ch) {
            const int64_t lo = base + S * ch / NCH, hi = base + S * (ch + 1) / NCH;
            std::vector<uint32_t> pend((size_t)nodes, kNone);
            for (int64_t i = lo; i < hi; ++i) {
                uint32_t& q = pend[pu[i]];
                if (q == kNone) q = (uint32_t)i;
                else { pL[i] = q; pL[q] = (uint32_t)i; q = kNone; }
            }
            for (int64_t u = 0; u < nodes; ++u)
                if (pend[u] != kNone) { leftL[ch].push_back(pend[u]); pend[u] = kNone; }
            for (int64_t i = lo; i < hi; ++i) {
                uint32_t& q = pend[pv[i]];
                if (q == kNone) q = (uint32_t)i;
                else { pR[i] = q; pR[q] = (uint32_t)i; q = kNone; }
            }
            for (int64_t u = 0; u < nodes; ++u)
                if (pend[u] != kNone) leftR[ch].push_back(pend[u]);
        }
        {
            std::vector<uint32_t> pend((size_t)nodes, kNone);
            for (int ch = 0; ch < NCH; ++ch)
                for (uint32_t i : leftL[ch]) {
                    uint32_t& q = pend[pu[i]];
                    if (q == kNone) q = i;
                    else { pL[i] = q; pL[q] = i; q = kNone; }
                }
            std::fill(pend.begin(), pend.end(), kNone);
            for (int ch = 0; ch < NCH; ++ch)
                for (uint32_t i : leftR[ch]) {
                    uint32_t& q = pend[pv[i]];
                    if (q == kNone) q = i;
                    else { pR[i] = q; pR[q] = i; q = kNone; }
                }
        }
        const double ms_pair = ms_since(t0);
        if ((int64_t)owner.size() < S) owner.resize((size_t)S);
        int32_t* own = owner.data() - base;              // indexed by absolute position
#pragma omp parallel for schedule(static)
        for (int64_t i = base; i < base + S; ++i) own[i] = -1;
        // segment id = t + T * (walk number of thread t): no shared counter
        struct Bound { uint32_t x, y; };
        std::vector<std::vector<Bound>> bounds(T);
        std::vector<std::vector<uint32_t>> segmin(T);    // smallest position a walk claimed
        std::vector<int32_t> walks(T, 0);
        auto claim = [&](uint32_t e, int32_t sid) {
            int32_t expect = -1;
            return __atomic_compare_exchange_n(&own[e], &expect, sid, false, __ATOMIC_RELAXED,
                                               __ATOMIC_RELAXED);
        };
        // one iteration per range t (not per OpenMP thread): correct whatever team size the
        // runtime grants (OMP_DYNAMIC, nested regions, thread limits)
#pragma omp parallel for schedule(static, 1)
        for (int t = 0; t < T; ++t) {
            const int64_t lo = base + S * t / T, hi = base + S * (t + 1) / T;
            std::vector<Bound>& bd = bounds[t];
            std::vector<uint32_t>& mins = segmin[t];
            int32_t w = 0;
            for (int64_t e0 = lo; e0 < hi; ++e0) {
                if (__atomic_load_n(&own[e0], __ATOMIC_RELAXED) != -1) continue;
                const int32_t sid = t + T * w;
                if (!claim((uint32_t)e0, sid)) continue;
                ++w;
                bit[e0] = 0;
                uint32_t mn = (uint32_t)e0;
                for (int dir = 0; dir < 2; ++dir) {       // 0: L first (forward), 1: R first
                    uint32_t cur = (uint32_t)e0;
                    while (true) {
                        const uint32_t a = dir == 0 ? pL[cur] : pR[cur];
                        if (!claim(a, sid)) { bd.push_back({cur, a}); break; }
                        bit[a] = bit[cur] ^ 1;
                        mn = a < mn ? a : mn;
                        const uint32_t b = dir == 0 ? pR[a] : pL[a];
                        if (!claim(b, sid)) { bd.push_back({a, b}); break; }
                        bit[b] = bit[a] ^ 1;
                        mn = b < mn ? b : mn;
                        cur = b;
                    }
                }
                mins.push_back(mn);
            }
            walks[t] = w;
        }
        const double ms_walk = ms_since(t0);
        // parity union-find over segments: flip[A] ^ flip[B] = (bit[x] == bit[y])
        int32_t maxw = 0;
        for (int t = 0; t < T; ++t) maxw = std::max(maxw, walks[t]);
        const int64_t nseg = (int64_t)T * maxw;
        std::vector<int32_t> parent((size_t)nseg);
        std::vector<uint8_t> par((size_t)nseg, 0);
        std::iota(parent.begin(), parent.end(), 0);
        auto find = [&](int32_t s, uint8_t& px) {
            uint8_t acc = 0;
            int32_t r0 = s;
            while (parent[r0] != r0) { acc ^= par[r0]; r0 = parent[r0]; }
            // path compression with parity
            uint8_t acc2 = acc;
            while (parent[s] != s) {
                const int32_t nx = parent[s];
                const uint8_t ps = par[s];
                parent[s] = r0;
                par[s] = acc2;
                acc2 ^= ps;
                s = nx;
            }
            px = acc;
            return r0;
        };
        for (int t = 0; t < T; ++t)
            for (const Bound& b : bounds[t]) {
                const int32_t A = own[b.x], B = own[b.y];
                if (A == B) continue;                     // closed inside one walk: consistent
                const uint8_t dd = (bit[b.x] == bit[b.y]) ? 1 : 0;
                uint8_t pa, pb;
                const int32_t ra = find(A, pa), rb = find(B, pb);
                if (ra != rb) { parent[ra] = rb; par[ra] = (uint8_t)(pa ^ pb ^ dd); }
            }
        // canonical polarity: in every cycle (component) the smallest position gets bit 0,
        // so the colouring does not depend on which walk happened to claim what
        std::vector<uint8_t> flip((size_t)nseg, 0);
        std::vector<uint32_t> cmin((size_t)nseg, kNone);
        std::vector<uint8_t> cbit((size_t)nseg, 0);
        std::vector<int32_t> root((size_t)nseg, -1);
        for (int t = 0; t < T; ++t)
            for (int32_t w = 0; w < walks[t]; ++w) {
                const int32_t s = t + T * w;
                uint8_t px;
                const int32_t rt = find(s, px);
                root[s] = rt;
                flip[s] = px;
                const uint32_t m = segmin[t][w];
                if (m < cmin[rt]) { cmin[rt] = m; cbit[rt] = (uint8_t)(bit[m] ^ px); }
            }
        for (int64_t s = 0; s < nseg; ++s)
            if (root[s] >= 0) flip[s] ^= cbit[root[s]];
#pragma omp parallel for schedule(static)
        for (int64_t i = base; i < base + S; ++i)
            if (flip[own[i]]) bit[i] ^= 1;
        const double ms_flip = ms_since(t0);
        // parallel stable partition (zeros first)
        std::vector<int64_t> zc(T + 1, 0);
#pragma omp parallel for schedule(static, 1)
        for (int t = 0; t < T; ++t) {
            const int64_t lo = base + S * t / T, hi = base + S * (t + 1) / T;
            int64_t z = 0;
            for (int64_t i = lo; i < hi; ++i) z += bit[i] == 0;
            zc[t + 1] = z;
        }
        for (int u = 0; u < T; ++u) zc[u + 1] += zc[u];
#pragma omp parallel for schedule(static, 1)
        for (int t = 0; t < T; ++t) {
            const int64_t lo = base + S * t / T, hi = base + S * (t + 1) / T;
            int64_t zp = base + zc[t], op = base + S / 2 + ((lo - base) - zc[t]);
            for (int64_t i = lo; i < hi; ++i) {
                const int64_t dst = bit[i] ? op++ : zp++;
                ord2[dst] = ord[i];
                pu2[dst] = pu[i];
                pv2[dst] = pv[i];
            }
        }
        if (verbose)
            std::fprintf(stderr, "  split_par S=%lld: pair %.1f walk %.1f flip %.1f total %.1f ms (segments %lld)\n",
                         (long long)S, ms_pair, ms_walk, ms_flip, ms_since(t0), (long long)nseg);
    }

    void run(int64_t nodes, int64_t d, int64_t E, const uint32_t* U, const uint32_t* V,
             uint32_t* colour, bool parallel) {
        if (d <= 1) {
            std::fill(colour, colour + E, 0u);
            return;
        }
        if ((int64_t)ord.size() < E) {
            ord.resize(E); ord2.resize(E); pu.resize(E); pu2.resize(E);
            pv.resize(E); pv2.resize(E); pL.resize(E); pR.resize(E); bit.resize(E);
        }
        for (int64_t i = 0; i < E; ++i) { ord[i] = (uint32_t)i; pu[i] = U[i]; pv[i] = V[i]; }
        const int levels = ilog2(d);
        static const bool verbose = std::getenv("PERM_PLANNER_VERBOSE") != nullptr;
        for (int lvl = 0; lvl < levels; ++lvl) {
            const int64_t G = int64_t(1) << lvl, S = E / G;
            auto tl = clk::now();
            // big groups: the chunked-pairing split (all threads inside one group). The choice
            // depends on S only, never on the thread count: every machine and every rank of a
            // sharded plan produces the same colouring.
            if (parallel && S >= (int64_t(1) << 20)) {
                for (int64_t g = 0; g < G; ++g) split_group_par(g * S, S, nodes);
            } else if (parallel && G > 1) {
#pragma omp parallel
                {
                    std::vector<uint32_t> pend(nodes);
#pragma omp for schedule(dynamic, 1)
                    for (int64_t g = 0; g < G; ++g) split_group(g * S, S, nodes, pend);
                }
            } else {
                std::vector<uint32_t> pend(nodes);
                for (int64_t g = 0; g < G; ++g) split_group(g * S, S, nodes, pend);
            }
            ord.swap(ord2); pu.swap(pu2); pv.swap(pv2);
            if (verbose && E >= (int64_t(1) << 20))
                std::fprintf(stderr, "euler level %d: G=%lld S=%lld %.1f ms\n", lvl, (long long)G,
                             (long long)S, ms_since(tl));
        }
        const int64_t per = E / d;   // a perfect matching per colour
        for (int64_t i = 0; i < E; ++i) colour[ord[i]] = (uint32_t)(i / per);
    }
};

// ---------------------------------------------------------------- conflict model

// Wavefronts of one 128-bit shared access by a warp: 4 phases of 8 lanes,
// each phase needs one wavefront per distinct 16-byte chunk in one bank group.
int wavefronts_v4(const int64_t* addr /*32 element addresses, 16B aligned*/) {
    int total = 0;
    for (int q = 0; q < 4; ++q) {
        int worst = 0;
        for (int bg = 0; bg < 8; ++bg) {
            int64_t seen[8];
            int cnt = 0;
            for (int l = 0; l < 8; ++l) {
                int64_t ch = addr[q * 8 + l] >> 2;
                if ((ch & 7) != bg) continue;
                bool dup = false;
                for (int u = 0; u < cnt; ++u) dup |= seen[u] == ch;
                if (!dup) seen[cnt++] = ch;
            }
            worst = std::max(worst, cnt);
        }
        total += std::max(worst, 1);
    }
    return (total + 3) / 4;
}

// Wavefronts of one 32-bit shared access by a warp.
int wavefronts_s(const int64_t* addr) {
    int worst = 0;
    for (int b = 0; b < 32; ++b) {
        int64_t seen[32];
        int cnt = 0;
        for (int l = 0; l < 32; ++l) {
            if ((addr[l] & 31) != b) continue;
            bool dup = false;
            for (int u = 0; u < cnt; ++u) dup |= seen[u] == addr[l];
            if (!dup) seen[cnt++] = addr[l];
        }
        worst = std::max(worst, cnt);
    }
    return std::max(worst, 1);
}

}  // namespace

void euler_split_colour(int64_t nodes, int64_t d, int64_t E, const uint32_t* U,
                        const uint32_t* V, uint32_t* colour, bool parallel) {
    EulerColourer ec;
    ec.run(nodes, d, E, U, V, colour, parallel);
}

// Mirrors the load/store loops of row_pass_kernel (kernels.cu): thread tid,
// iteration it handles the 4-element vector f = 4*(tid + T*it).
int simulate_conflicts(const RowPass& rp, const PhaseGeom& g, bool input_side) {
    const IoMode& m = input_side ? rp.in : rp.out;
    const int64_t L = g.L, h = rp.h, T = rp.threads, total = h * L;
    const int64_t iters = total / (4 * T);
    int worst = 1;
    int64_t addr[32];
    for (int64_t it = 0; it < iters; ++it) {
        for (int64_t w0 = 0; w0 < T; w0 += 32) {
            if (!m.cross) {
                for (int l = 0; l < 32; ++l) {
                    int64_t f = 4 * (w0 + l + T * it);
                    int64_t K = f / (h * m.w), line = (f / m.w) % h, kk = f % m.w;
                    addr[l] = line * rp.Ls + K * m.w + kk;
                }
                worst = std::max(worst, wavefronts_v4(addr));
            } else {
                for (int j = 0; j < 4; ++j) {
                    for (int l = 0; l < 32; ++l) {
                        int64_t f = 4 * (w0 + l + T * it);
                        int64_t pos = f / h, line = f % h + j;
                        addr[l] = line * rp.Ls + pos;
                    }
                    worst = std::max(worst, wavefronts_s(addr));
                }
            }
        }
    }
    return worst;
}

namespace {

void choose_threads(RowPass& rp, int64_t L) {
    const int64_t total = rp.h * L;
    int ept = 16;
    while (total / ept > 512 && ept < 64) ept *= 2;
    while (total / ept < 64 && ept > 4) ept /= 2;
    rp.ept = ept;
    rp.threads = (int32_t)(total / ept);
}

void choose_pad(RowPass& rp, const PhaseGeom& g) {
    const bool needs_v4 = !rp.in.cross || !rp.out.cross;
    int best_pad = 0, best = 1 << 30;
    for (int pad = 0; pad < 32; ++pad) {
        if (needs_v4 && (pad & 3)) continue;
        rp.Ls = g.L + pad;
        int ci = simulate_conflicts(rp, g, true);
        int co = simulate_conflicts(rp, g, false);
        if (ci + co < best) { best = ci + co; best_pad = pad; }
        if (best == 2) break;
    }
    rp.Ls = g.L + best_pad;
    rp.conflicts_in = simulate_conflicts(rp, g, true);
    rp.conflicts_out = simulate_conflicts(rp, g, false);
}

IoMode runs(int64_t w, int64_t strideK, int64_t cta_stride) {
    IoMode m;
    m.cross = 0; m.w = (int32_t)w; m.strideK = strideK; m.cta_stride = cta_stride;
    return m;
}
IoMode cross(int64_t blockP, int64_t strideP, int64_t cta_stride) {
    IoMode m;
    m.cross = 1; m.blockP = (int32_t)blockP; m.strideP = strideP; m.cta_stride = cta_stride;
    return m;
}

}  // namespace

// ------------------------------------------------------------------ TLC layout

// Colour every tile's bank graph (edge (src mod 32, dst mod 32) per element; the graph
// is (HL/32)-regular because A and B are dense) and pack the entries in the TLC
// bitstream format (plan.hpp TlcPass): colour = warp-round q, lane = source bank.
// enum_tile(T, src, dst, tval) lists tile T's elements. W must be zeroed, sized
// ntiles * tile_words. `bad` is set when an entry does not decode to its dst.
template <class Enum>
int colour_and_pack(const TlcPass& tp, bool gpu, Enum&& enum_tile, U32Buf& Wbuf, int& bad,
                    std::string& err) {
    const int64_t HL = tp.HL;
    const int E = tp.E, ept = tp.ept, nwords = tp.nwords;
    const TlcDecode dec = tp.dec;
    Wbuf.assign((size_t)(tp.ntiles * tp.tile_words), 0u);
    uint32_t* W = Wbuf.data();
    std::vector<uint16_t> gcol;
    if (gpu) {
        // every tile's bank graph at once on the device (vertex (tile, offset mod 32))
        const int64_t N = tp.ntiles * HL;
        U16Buf ks((size_t)N), kd((size_t)N);
#pragma omp parallel
        {
            std::vector<uint32_t> src((size_t)HL), dst((size_t)HL), tval((size_t)HL);
#pragma omp for schedule(static)
            for (int64_t T = 0; T < tp.ntiles; ++T) {
                enum_tile(T, src.data(), dst.data(), tval.data());
                for (int64_t x = 0; x < HL; ++x) {
                    ks[T * HL + x] = (uint16_t)src[x];
                    kd[T * HL + x] = (uint16_t)dst[x];
                }
            }
        }
        gcol.resize((size_t)N);
        GpuPlanStats gs;
        const cudaError_t ce = gpu_bank_colour(ks.data(), kd.data(), N, tp.logHL, gcol.data(), &gs);
        if (ce != cudaSuccess) {
            err = std::string("GPU planner (TLC bank colouring): ") + cudaGetErrorString(ce);
            return ce == cudaErrorMemoryAllocation ? PERM_ENOMEM : PERM_ECUDA;
        }
    }
#pragma omp parallel reduction(| : bad)
    {
        EulerColourer ec;
        std::vector<uint32_t> U((size_t)HL), V((size_t)HL), col((size_t)HL), src((size_t)HL), dst((size_t)HL),
            tval((size_t)HL);
#pragma omp for schedule(dynamic, 1)
        for (int64_t T = 0; T < tp.ntiles; ++T) {
            enum_tile(T, src.data(), dst.data(), tval.data());
            if (!gcol.empty()) {
                for (int64_t x = 0; x < HL; ++x) col[x] = gcol[T * HL + x];
            } else {
                for (int64_t x = 0; x < HL; ++x) { U[x] = src[x] & 31; V[x] = dst[x] & 31; }
                ec.run(kW, HL / kW, HL, U.data(), V.data(), col.data(), false);
            }
            uint32_t* Wt = W + T * tp.tile_words;
            for (int64_t x = 0; x < HL; ++x) {
                const int64_t q = col[x];                 // warp-round
                const int64_t lane = src[x] & 31;         // lane = source bank
                const int64_t pw = q / ept, m = q % ept;
                const uint32_t t = tval[x];
                if (tlc_dst(dec, t, src[x]) != dst[x]) bad = 1;   // decode self-check
                const uint64_t entry = ((uint64_t)(src[x] >> 5) << dec.lt) | t;
                const int64_t bit = m * E;
                const int64_t w = bit >> 5, off = bit & 31;
                const uint64_t sh = entry << off;
                uint32_t* base = Wt + (pw * nwords) * 32 + lane;
                base[w * 32] |= (uint32_t)sh;
                if (off + E > 32) base[(w + 1) * 32] |= (uint32_t)(sh >> 32);
            }
        }
    }
    return PERM_OK;
}



// Word offsets of the element (line, position) of tile T in the A / B buffers of
// each TLC pass (see plan.hpp and DESIGN.md §5):
//   X1 = [K][i][k_in] (K < c/h2, i < r, k_in < h2)   X2 = [I'][K][i_in'][k_in]
//   pass 1: src = i_in*c + j,                     dst = ((k/h2)*h1 + i_in)*h2 + k%h2
//   pass 2: src = i*h2 + k_in,                    dst = i'*h2 + k_in
//   pass 3: src = ((k/h2)*h3 + i_in)*h2 + k%h2,   dst = i_in*c + k'
int build_tlc(HostPlan& P, const U16Buf* phi, const perm_plan_options* opt,
              std::string& err) {
    const int64_t r = P.r, c = P.c;
    P.layout = 3;
    const int stages_opt = (opt && opt->stages > 0) ? opt->stages : 0;
    int64_t hs[3];
    for (int f = 0; f < 3; ++f) {
        const int64_t L = P.ph[f].L, lines_f = P.ph[f].lines;
        // default tiles: 8192 words up to 2^24 (pass 2 keeps h2 >= 4 for 16-byte TMA box rows,
        // so 16384 words at 2^24), 16384 words at 2^25. The transposed chunks are h1*h2 words:
        // 16 at 2^22, 8 (32 bytes) at 2^23 - 2^25. Smaller row tiles at 2^23 / 2^24 measured
        // 41.0 / 90.3 us against 47.5 / 98.0 us with h1 = h3 = 4 (profiles/r02_ab_mid.jsonl).
        // Up to 2^19, 8192-word tiles leave SMs idle (32 / 64 tiles per pass at 2^18 / 2^19 on
        // 148 SMs): 4096-word tiles, 14.7 -> 13.3 us and 15.5 -> 13.4 us (profiles/r02_ab_small.jsonl).
        // At 2^21 4096-word tiles (h = 2, 4, 2; 512 tiles per pass) beat 8192-word ones (h = 4,
        // 8, 4): 19.44 -> 18.99 us (profiles/r02b_tiles_21.log); equal at 2^20.
        const int64_t T = (P.k <= 19 || P.k == 21) ? 4096 : (P.k <= 24 ? 8192 : 16384);
        int64_t h = (opt && (&opt->h1)[f] > 0)
                        ? (&opt->h1)[f]
                        : (P.k <= 24 ? std::max<int64_t>(f == 1 ? 4 : 2, T / L) : std::max<int64_t>(1, T / L));
        h = std::min(h, lines_f);
        // h2 is the inner dimension of the TMA tensor boxes (>= 16 bytes)
        if (h < (f == 1 ? 4 : 1) || (h & (h - 1)) || lines_f % h) {
            err = "TLC layout: h must be a power of two (h2 >= 4)";
            return PERM_EINVAL;
        }
        hs[f] = h;
    }
    const int64_t h1 = hs[0], h2 = hs[1], h3 = hs[2];
    for (int f = 0; f < 3; ++f) {
        TlcPass& tp = P.tp[f];
        tp.h = (int32_t)hs[f];
        tp.HL = (int32_t)(hs[f] * P.ph[f].L);
        tp.logHL = ilog2(tp.HL);
        tp.ept = tp.HL / kTlcPerm;
        if (tp.ept != 8 && tp.ept != 16 && tp.ept != 32) {
            err = "TLC layout: tile must hold 4096, 8192 or 16384 elements (h * L)";
            return PERM_EINVAL;
        }
        // entry format (plan.hpp TlcDecode): compact when a kernel is compiled for its width
        const int logL = P.ph[f].logL;
        const int cmp_opt = opt ? opt->sched_format : 0;
        const int Ec = tp.logHL - 5 + logL;
        TlcDecode d;
        // the kernels take pass 2's and pass 3's line index from the lane alone (free decode):
        // needs h2 <= 32 (pass 2) and h2 * h3 <= 32 (pass 3)
        const bool lane_line = (f != 1 || hs[1] <= kW) && (f != 2 || hs[1] * hs[2] <= kW);
        // default (0): compact from n = 2^23 on (B200, cold L2: 2^23 41.7 -> 40.6 us, 2^24 85.0 ->
        // 84.4, 2^25 185.5 -> 181.3; equal at 2^22, profiles/r02b_compact_ab.log); -1: full
        const bool fused_req = opt && opt->fuse > 0;
        const bool want_compact = cmp_opt > 0 || (cmp_opt == 0 && r * c >= (int64_t(1) << 23));
        if (want_compact && !fused_req && tlc_compact_supported(tp.ept, Ec) && lane_line) {
            const int lh1 = ilog2(hs[0]), lh2 = ilog2(hs[1]), lc = ilog2(P.c);
            d.lt = logL;
            if (f == 0) {          // dst = ((k/h2)*h1 + i_in)*h2 + k%h2, i_in = src >> log c
                d.s1 = lh2; d.s2 = lh1 + lh2; d.s4 = lc; d.m2 = (uint32_t)hs[0] - 1; d.s3 = lh2;
                d.m1 = (uint32_t)hs[1] - 1;
            } else if (f == 1) {   // dst = i'*h2 + k_in, k_in = src mod h2
                d.s1 = 0; d.s2 = lh2; d.s4 = 0; d.m2 = (uint32_t)hs[1] - 1; d.s3 = 0; d.m1 = 0;
            } else {               // dst = i_in*c + k', i_in = (src >> log h2) mod h3
                d.s1 = lc; d.s2 = 0; d.s4 = lh2; d.m2 = (uint32_t)hs[2] - 1; d.s3 = lc;
                d.m1 = (uint32_t)P.c - 1;
            }
            tp.E = Ec;
        } else {
            d.lt = tp.logHL;       // full format: dst = t
            tp.E = 2 * tp.logHL - 5;
        }
        tp.dec = d;
        tp.nwords = (tp.ept * tp.E + 31) / 32;
        tp.ntiles = P.ph[f].lines / hs[f];
        tp.tile_words = (int64_t)(kTlcPerm / 32) * tp.nwords * 32;
        tp.out_kind = f == 0 ? 1 : (f == 1 ? 2 : 0);
        // separate rings: A slots take TMA loads (a CTA's whole share of tiles in flight
        // when it fits), B slots hold permuted tiles until their TMA store has read them
        const int64_t slot = (int64_t)tp.HL * 4;
        const int64_t budget = 220 * 1024;
        const int nb = slot * 4 <= budget ? 2 : 1;
        const int64_t fit = budget / slot - nb;
        int st = stages_opt ? stages_opt : (int)std::min<int64_t>(6, fit);
        if (st < 1 || (st + nb) * slot > budget) { err = "TLC layout: stages do not fit in shared memory"; return PERM_EINVAL; }
        tp.stages = st;
        tp.bslots = nb;
        // keep the generic RowPass view consistent for info/describe
        RowPass& rp = P.rp[f];
        rp.phase = f; rp.h = tp.h; rp.ctas = tp.ntiles; rp.tma = 3; rp.stages = st;
        rp.ept = tp.ept; rp.threads = 64 + kTlcPerm; rp.Ls = P.ph[f].L;
    }
    // TMA tensor stores need 16-byte rows: h2 * 4 >= 16 (h2 >= 4 holds)
    for (int f = 0; f < 3; ++f) {
        const TlcPass& tp = P.tp[f];
        const uint16_t* ph = phi[f].data();
        const int64_t h = tp.h;
        const TlcDecode dec = tp.dec;
        const bool full = dec.lt == tp.logHL && dec.s2 == 0 && dec.s3 == 0 && dec.m1 == 0;
        // element x of tile T: source offset in A, destination offset in B, entry payload
        auto enum_tile = [&](int64_t T, uint32_t* src, uint32_t* dst, uint32_t* tval) {
                int64_t e = 0;
                if (f == 0) {
                    for (int64_t i_in = 0; i_in < h; ++i_in)
                        for (int64_t j = 0; j < c; ++j, ++e) {
                            const int64_t kk = ph[(T * h + i_in) * c + j];
                            src[e] = (uint32_t)(i_in * c + j);
                            dst[e] = (uint32_t)(((kk / h2) * h1 + i_in) * h2 + kk % h2);
                            tval[e] = full ? dst[e] : (uint32_t)kk;
                        }
                } else if (f == 1) {
                    for (int64_t k_in = 0; k_in < h; ++k_in)
                        for (int64_t i = 0; i < r; ++i, ++e) {
                            const int64_t ip = ph[(T * h + k_in) * r + i];
                            src[e] = (uint32_t)(i * h2 + k_in);
                            dst[e] = (uint32_t)(ip * h2 + k_in);
                            tval[e] = full ? dst[e] : (uint32_t)ip;
                        }
                } else {
                    for (int64_t i_in = 0; i_in < h; ++i_in)
                        for (int64_t kk = 0; kk < c; ++kk, ++e) {
                            const int64_t kp = ph[(T * h + i_in) * c + kk];
                            src[e] = (uint32_t)(((kk / h2) * h3 + i_in) * h2 + kk % h2);
                            dst[e] = (uint32_t)(i_in * c + kp);
                            tval[e] = full ? dst[e] : (uint32_t)kp;
                        }
                }
        };
        int bad = 0;
        const int st = colour_and_pack(tp, opt && opt->gpu_planner > 0, enum_tile, P.sched[f], bad, err);
        if (st != PERM_OK) return st;
        if (bad) { err = "TLC layout: internal error (entry decode mismatch)"; return PERM_ECUDA; }
    }
    return PERM_OK;
}

// ------------------------------------------------------------------ TLC through the half-line ring
//
// 2^26 / 2^27 (layout 5): the TLC passes (tile-level colouring, transposes absorbed into the
// intermediates' chunk layouts) with 32768-word tiles, so that the transposed
// chunks are 16 / 8 words; a tile of 128 KiB is permuted in place through the three 64 KiB
// half-tile slots of row_pass_split_stg_kernel (the L = 32768 row-pass machinery), whose
// stores write the two halves of the tile's output order as X1 / X2 tensor-store chunks.
// Schedules: every tile's bank graph (src mod 32, dst mod 32) coloured, packed in the dense
// per-round format of a 32768-word "line" (entry (src >> 5) << 15 | dst, E = 25 bits).
int build_tlc_ring(HostPlan& P, const U16Buf* phi, const perm_plan_options* opt, std::string& err) {
    const int64_t r = P.r, c = P.c;
    constexpr int64_t HL = 32768;
    int64_t hs[3];
    for (int f = 0; f < 3; ++f) {
        const int64_t L = P.ph[f].L;
        const int64_t h = (opt && (&opt->h1)[f] > 0) ? (&opt->h1)[f] : HL / L;
        if (h * L != HL || (h & (h - 1)) || P.ph[f].lines % h || (f == 1 && h < 4)) {
            err = "TLC ring layout: tiles must hold 32768 words (h * L), h2 >= 4";
            return PERM_EINVAL;
        }
        hs[f] = h;
    }
    const int64_t h1 = hs[0], h2 = hs[1], h3 = hs[2];
    if (h1 * h2 < 4 || h3 * h2 < 4) { err = "TLC ring layout: transposed chunks under 16 bytes"; return PERM_EINVAL; }
    P.layout = 5;
    P.passes = 3;
    for (int f = 0; f < 3; ++f) {
        TlcPass& tp = P.tp[f];
        tp = TlcPass{};
        tp.h = (int32_t)hs[f];
        tp.HL = (int32_t)HL;
        tp.logHL = 15;
        tp.E = 25;
        tp.ntiles = P.ph[f].lines / hs[f];
        tp.out_kind = f == 0 ? 1 : (f == 1 ? 2 : 0);
        tp.dec.lt = 15;
        // the tile is the ring kernel's "line": one 32768-word line per CTA step
        PhaseGeom& g = P.ph[f];
        g.lines = tp.ntiles;
        g.L = (int32_t)HL;
        g.logL = 15;
        g.E = 25;
        g.epw = 64 / g.E;
        g.w64 = (kW + g.epw - 1) / g.epw;
        g.dense = 1;
        g.wpl = (HL / kW) * g.E;
        g.words = g.lines * g.wpl;
        RowPass& rp = P.rp[f];
        rp = RowPass{};
        rp.phase = f; rp.h = 1; rp.ctas = tp.ntiles;
        rp.in = IoMode{}; rp.out = IoMode{};
        rp.in.w = (int32_t)HL; rp.out.w = (int32_t)HL;
        rp.in.cta_stride = HL; rp.out.cta_stride = HL;
        rp.tma = 1; rp.sg = 1; rp.split = 1; rp.split_stg = 1; rp.stages = 3;
        rp.threads = 512; rp.ept = (int32_t)(HL / 512); rp.Ls = (int32_t)HL;
    }
    for (int f = 0; f < 3; ++f) {
        const TlcPass& tp = P.tp[f];
        const PhaseGeom& g = P.ph[f];
        const uint16_t* ph = phi[f].data();
        const int64_t h = tp.h;
        // element x of tile T: source offset in the tile (input order), destination offset
        // (output order) -- the TLC layouts of build_tlc
        auto enum_tile = [&](int64_t T, uint32_t* src, uint32_t* dst) {
            int64_t e = 0;
            if (f == 0) {
                for (int64_t i_in = 0; i_in < h; ++i_in)
                    for (int64_t j = 0; j < c; ++j, ++e) {
                        const int64_t kk = ph[(T * h + i_in) * c + j];
                        src[e] = (uint32_t)(i_in * c + j);
                        dst[e] = (uint32_t)(((kk / h2) * h1 + i_in) * h2 + kk % h2);
                    }
            } else if (f == 1) {
                for (int64_t k_in = 0; k_in < h; ++k_in)
                    for (int64_t i = 0; i < r; ++i, ++e) {
                        const int64_t ip = ph[(T * h + k_in) * r + i];
                        src[e] = (uint32_t)(i * h2 + k_in);
                        dst[e] = (uint32_t)(ip * h2 + k_in);
                    }
            } else {
                for (int64_t i_in = 0; i_in < h; ++i_in)
                    for (int64_t kk = 0; kk < c; ++kk, ++e) {
                        const int64_t kp = ph[(T * h + i_in) * c + kk];
                        src[e] = (uint32_t)(((kk / h2) * h3 + i_in) * h2 + kk % h2);
                        dst[e] = (uint32_t)(i_in * c + kp);
                    }
            }
        };
        std::vector<uint16_t> gcol;
        if (opt && opt->gpu_planner > 0) {
            const int64_t N = tp.ntiles * HL;
            U16Buf ks((size_t)N), kd((size_t)N);
#pragma omp parallel
            {
                std::vector<uint32_t> src((size_t)HL), dst((size_t)HL);
#pragma omp for schedule(static)
                for (int64_t T = 0; T < tp.ntiles; ++T) {
                    enum_tile(T, src.data(), dst.data());
                    for (int64_t x = 0; x < HL; ++x) {
                        ks[T * HL + x] = (uint16_t)src[x];
                        kd[T * HL + x] = (uint16_t)dst[x];
                    }
                }
            }
            gcol.resize((size_t)N);
            GpuPlanStats gs;
            const cudaError_t ce = gpu_bank_colour(ks.data(), kd.data(), N, 15, gcol.data(), &gs);
            if (ce != cudaSuccess) {
                err = std::string("GPU planner (TLC ring bank colouring): ") + cudaGetErrorString(ce);
                return ce == cudaErrorMemoryAllocation ? PERM_ENOMEM : PERM_ECUDA;
            }
        }
        P.sched[f].assign((size_t)g.words + 4, 0u);
        uint32_t* W = P.sched[f].data();
#pragma omp parallel
        {
            EulerColourer ec;
            std::vector<uint32_t> U((size_t)HL), V((size_t)HL), col((size_t)HL), src((size_t)HL), dst((size_t)HL);
#pragma omp for schedule(dynamic, 1)
            for (int64_t T = 0; T < tp.ntiles; ++T) {
                enum_tile(T, src.data(), dst.data());
                if (!gcol.empty()) {
                    for (int64_t x = 0; x < HL; ++x) col[x] = gcol[T * HL + x];
                } else {
                    for (int64_t x = 0; x < HL; ++x) { U[x] = src[x] & 31; V[x] = dst[x] & 31; }
                    ec.run(kW, HL / kW, HL, U.data(), V.data(), col.data(), false);
                }
                for (int64_t x = 0; x < HL; ++x) {
                    const uint64_t entry = ((uint64_t)(src[x] >> 5) << 15) | dst[x];
                    pack_entry(W, g, T, (int64_t)col[x] * kW + (src[x] & 31), entry);
                }
            }
        }
    }
    return PERM_OK;
}

// ------------------------------------------------------------------ cluster path
//
// n <= 2^18 (NEXT-4: the whole array fits on chip): ONE launch of one
// thread-block cluster of C blocks (DESIGN.md §5 "cluster path"). Block g holds
// S = n/C words and owns rows [g*r_l, (g+1)*r_l) in phases 1 and 3, columns
// [g*c_l, (g+1)*c_l) in phase 2 (r_l = r/C, c_l = c/C). Each phase is one
// tile-coloured permute in the block's shared memory from its A buffer (input
// order) to its B buffer (output order); the column phase's two transposes
// (Lemma 8) become two exchanges of uniform Bw = r_l*c_l-word blocks over
// distributed shared memory -- the row-sharded multi-GPU scheme
// with DSMEM for NVLink:
//   phase 1: A = rows of a (i_l*c + j);  B = send blocks, (i, k) at (k/c_l)*Bw + (k%c_l)*r_l + i%r_l
//   exchange: send block q of block g -> block q's A at [g*Bw, (g+1)*Bw)
//   phase 2: A = [sender][k_in][i_l];    B = send blocks, (i', k) at (i'/r_l)*Bw + (i'%r_l)*c_l + k%c_l
//   exchange
//   phase 3: A = [sender][i'_l][k_in];   B = rows of b (i'_l*c + k')
int build_cluster(HostPlan& P, const U16Buf* phi, const perm_plan_options* opt, std::string& err) {
    const int64_t n = P.n, r = P.r, c = P.c;
    int64_t C = (opt && opt->cluster > 0) ? opt->cluster : 16;
    while (C > 1 && n / C > 16384) C *= 2;
    const int64_t S = n / C;
    if (C < 2 || C > 16 || (C & (C - 1)) || r % C || c % C || S < 2048 || S > 16384 ||
        (r / C) * (c / C) < 4) {
        err = "cluster path: needs a power-of-two cluster of 2..16 blocks with 2048..16384 words "
              "per block (n = 2^15..2^18) and r, c divisible by it";
        return PERM_EUNSUPPORTED;
    }
    P.passes = 2;
    P.layout = 4;
    P.cluster = (int32_t)C;
    const int64_t rl = r / C, cl = c / C, Bw = rl * cl;
    for (int f = 0; f < 3; ++f) {
        TlcPass& tp = P.tp[f];
        tp.h = (int32_t)(f == 1 ? cl : rl);
        tp.HL = (int32_t)S;
        tp.logHL = ilog2(S);
        tp.ept = tp.HL / kTlcPerm;
        tp.E = 2 * tp.logHL - 5;
        tp.dec = TlcDecode{};
        tp.dec.lt = tp.logHL;            // full format: entry = ((src >> 5) << log S) | dst
        tp.nwords = (tp.ept * tp.E + 31) / 32;
        tp.ntiles = C;
        tp.tile_words = (int64_t)(kTlcPerm / 32) * tp.nwords * 32;
        tp.stages = 0;
        tp.bslots = 0;
        RowPass& rp = P.rp[f];
        rp.phase = f; rp.h = tp.h; rp.ctas = C; rp.ept = tp.ept; rp.threads = kTlcPerm; rp.Ls = P.ph[f].L;
    }
    for (int f = 0; f < 3; ++f) {
        const TlcPass& tp = P.tp[f];
        const uint16_t* ph = phi[f].data();
        auto enum_tile = [&](int64_t g, uint32_t* src, uint32_t* dst, uint32_t* tval) {
            for (int64_t s = 0; s < S; ++s) {
                int64_t d;
                if (f == 0) {
                    const int64_t i_l = s / c, i = g * rl + i_l;
                    const int64_t k = ph[i * c + s % c];
                    d = (k / cl) * Bw + (k % cl) * rl + i_l;
                } else if (f == 1) {
                    const int64_t sender = s / Bw, rem = s % Bw;
                    const int64_t k_in = rem / rl, i = sender * rl + rem % rl;
                    const int64_t ip = ph[(g * cl + k_in) * r + i];
                    d = (ip / rl) * Bw + (ip % rl) * cl + k_in;
                } else {
                    const int64_t sender = s / Bw, rem = s % Bw;
                    const int64_t ip_l = rem / cl, k = sender * cl + rem % cl;
                    const int64_t kp = ph[(g * rl + ip_l) * c + k];
                    d = ip_l * c + kp;
                }
                src[s] = (uint32_t)s;
                dst[s] = (uint32_t)d;
                tval[s] = (uint32_t)d;
            }
        };
        int bad = 0;
        const int st = colour_and_pack(tp, opt && opt->gpu_planner > 0, enum_tile, P.sched[f], bad, err);
        if (st != PERM_OK) return st;
        if (bad) { err = "cluster path: internal error (entry decode mismatch)"; return PERM_ECUDA; }
    }
    return PERM_OK;
}

int build_host_plan(const int32_t* p, int64_t n, int32_t eb, const perm_plan_options* opt,
                    HostPlan& P, std::string& err) {
    if (!p || n <= 0) { err = "null p or n <= 0"; return PERM_EINVAL; }
    if (eb == 8) {
        // 8-byte elements (Table II(b)): element i is the word pair (2i, 2i+1);
        // permuting it to P(i) is the word permutation P'(2i + h) = 2P(i) + h, scheduled
        // like any other (reading #10).
        if (n > (int64_t(1) << 29)) { err = "n must be <= 2^29 for 8-byte elements"; return PERM_EUNSUPPORTED; }
        std::vector<uint8_t> seen((size_t)n, 0);
        for (int64_t i = 0; i < n; ++i) {
            const int32_t v = p[i];
            if (v < 0 || v >= n || seen[v]) {
                err = "p is not a permutation: entry " + std::to_string(i) + " = " + std::to_string(v);
                return PERM_ENOTPERM;
            }
            seen[v] = 1;
        }
        std::vector<int32_t> p2((size_t)(2 * n));
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) {
            p2[2 * i] = 2 * p[i];
            p2[2 * i + 1] = 2 * p[i] + 1;
        }
        const int st = build_host_plan(p2.data(), 2 * n, 4, opt, P, err);
        P.user_eb = 8;
        P.user_n = n;
        return st;
    }
    if (eb != 4) { err = "elem_bytes must be 4 or 8"; return PERM_EUNSUPPORTED; }
    P.user_eb = 4;
    P.user_n = n;
    const int k = ilog2(n);
    if ((int64_t(1) << k) != n || k < 10 || k > 30) {
        err = "n must be a power of two in [2^10, 2^30]";
        return PERM_EUNSUPPORTED;
    }
    // 1. validate: bijection onto [0, n) -- a parallel pass over an atomic bitmap,
    //    then (only when it fails) the serial pass that names the first bad entry
    bool valid = true;
    {
        std::vector<std::atomic<uint64_t>> bits((size_t)((n + 63) / 64));
#pragma omp parallel for schedule(static)
        for (int64_t w = 0; w < (int64_t)bits.size(); ++w) bits[w].store(0, std::memory_order_relaxed);
        int bad = 0;
#pragma omp parallel for schedule(static) reduction(| : bad)
        for (int64_t i = 0; i < n; ++i) {
            const int32_t v = p[i];
            if (v < 0 || v >= n) { bad = 1; continue; }
            const uint64_t m = uint64_t(1) << (v & 63);
            if (bits[v >> 6].fetch_or(m, std::memory_order_relaxed) & m) bad = 1;
        }
        valid = !bad;
    }
    if (!valid) {
        std::vector<uint8_t> seen((size_t)n, 0);
        for (int64_t i = 0; i < n; ++i) {
            const int32_t v = p[i];
            if (v < 0 || v >= n || seen[v]) {
                err = "p is not a permutation: entry " + std::to_string(i) + " = " +
                      std::to_string(v);
                return PERM_ENOTPERM;
            }
            seen[v] = 1;
        }
    }
    {
        // D_w(P) (L389-L401): distinct address groups of b written by each warp of 32
        int64_t dw = 0;
#pragma omp parallel for reduction(+ : dw) schedule(static)
        for (int64_t wj = 0; wj < n / kW; ++wj) {
            uint32_t g[kW];
            for (int x = 0; x < kW; ++x) g[x] = (uint32_t)p[wj * kW + x] >> 5;
            std::sort(g, g + kW);
            int64_t d = 1;
            for (int x = 1; x < kW; ++x) d += g[x] != g[x - 1];
            dw += d;
        }
        P.distribution = dw;
        const int dopt = opt ? opt->direct : 0;
        if (dopt > 0 || (dopt == 0 && dw <= 2 * n / kW)) {
            // D_w(P^-1) = D_w(P): both count the distinct (warp block of sources, address
            // group of destinations) pairs, so the S-designated kernel b[i] = a[q[i]]
            // (L373) reads as few groups as the D-designated one writes, and its writes
            // are whole sectors (the scatter's partial-sector writes cost 21 vs 12 us for
            // the shuffle at n = 2^22, profiles/bench_r01r.json s_designated_us).
            // direct = 2 keeps the D-designated kernel (A/B).
            // direct = 3 when P moves whole aligned 32-word blocks in order (identity,
            // block permutations): only the n/32-entry block map of P^-1 is read
            bool blocks = dopt <= 0;
            if (blocks) {
                int bad = 0;
#pragma omp parallel for schedule(static) reduction(| : bad)
                for (int64_t i = 0; i < n; ++i)
                    bad |= ((p[i] & (kW - 1)) != (i & (kW - 1))) |
                           ((p[i] - (i & (kW - 1))) != p[i & ~int64_t(kW - 1)]);
                blocks = !bad;
            }
            P.direct = blocks ? 3 : dopt == 2 ? 2 : 1;
            P.p_copy.resize((size_t)(blocks ? n / kW : n));
            if (P.direct == 3) {
                int32_t* qb = P.p_copy.data();
#pragma omp parallel for schedule(static)
                for (int64_t j = 0; j < n / kW; ++j) qb[p[j * kW] / kW] = (int32_t)j;
            } else if (P.direct == 2) {
                P.p_copy.assign(p, p + n);
            } else {
                int32_t* q = P.p_copy.data();
#pragma omp parallel for schedule(static)
                for (int64_t i = 0; i < n; ++i) q[p[i]] = (int32_t)i;
            }
        }
    }
    P.n = n; P.eb = eb; P.k = k;
    if (P.direct) {
        // low-distribution shortcut: perm_apply runs one kernel on p_copy, so no colouring,
        // schedule or scratch is built (direct = -1 keeps the scheduled passes for A/B runs)
        const int lc = k - k / 2;
        P.r = int64_t(1) << (k - lc);
        P.c = int64_t(1) << lc;
        P.passes = 0;
        return PERM_OK;
    }
    // view r x c (L603: "not restricted to a square matrix"); default c = 2^ceil(k/2)
    // n = 2^29 (5 passes): c = 2^14, r = 2^15, so the two row phases run on 16384-word
    // lines (schedule-from-global slots) and only the column phase on 32768-word lines
    // (half-line ring) -- the other way round it is two slow passes and one fast one
    const int logc_auto = (k == 29 && !(opt && opt->passes == 3)) ? 14 : k - k / 2;
    const int logc = (opt && opt->log2c > 0) ? opt->log2c : logc_auto, logr = k - logc;
    if (logc < 5 || logr < 5) { err = "view: log2c must leave r, c >= 32"; return PERM_EINVAL; }
    P.r = int64_t(1) << logr;
    P.c = int64_t(1) << logc;
    const int64_t r = P.r, c = P.c;
#ifdef _OPENMP
    P.threads_used = omp_get_max_threads();
#endif

    // 2-3. row-level colouring
    auto t0 = clk::now();
    const bool gpu = opt && opt->gpu_planner > 0;
    P.gpu_planner = gpu ? 1 : 0;
    P.kappa.resize((size_t)n);
    if (gpu) {
        GpuPlanStats gs;
        const cudaError_t ce = gpu_row_colour(p, n, logc, P.kappa.data(), &gs);
        if (ce != cudaSuccess) {
            err = std::string("GPU planner (row colouring): ") + cudaGetErrorString(ce);
            return ce == cudaErrorMemoryAllocation ? PERM_ENOMEM : PERM_ECUDA;
        }
    } else {
        std::vector<uint32_t> colour((size_t)n);
        {
            std::vector<uint32_t> U((size_t)n), V((size_t)n);
#pragma omp parallel for schedule(static)
            for (int64_t x = 0; x < n; ++x) {
                U[x] = (uint32_t)(x >> logc);
                V[x] = (uint32_t)((uint32_t)p[x] >> logc);
            }
            EulerColourer ec;
            ec.run(r, c, n, U.data(), V.data(), colour.data(), true);
        }
#pragma omp parallel for schedule(static)
        for (int64_t x = 0; x < n; ++x) P.kappa[x] = (uint16_t)colour[x];
    }
    P.ms_colour = ms_since(t0);

    // 4. phase permutations as per-line arrays (uint16: every L <= 2^15)
    t0 = clk::now();
    U16Buf phi[3];
    for (auto& v : phi) v.resize((size_t)n);
#pragma omp parallel for schedule(static)
    for (int64_t x = 0; x < n; ++x) {
        const int64_t i = x >> logc;
        const uint32_t kk = P.kappa[x];
        const uint32_t dest = (uint32_t)p[x];
        const uint32_t drow = dest >> logc, dcol = dest & (uint32_t)(c - 1);
        phi[0][x] = (uint16_t)kk;                               // Phi1_i(j) = kappa(x)
        phi[1][(int64_t)kk * r + i] = (uint16_t)drow;           // Phi2_k(i) = P(x) div c
        phi[2][(int64_t)drow * c + kk] = (uint16_t)dcol;        // Phi3_i'(k) = P(x) mod c
    }
    // pass structure
    int passes = opt ? opt->passes : 0;
    // measured on B200: fused CTA to 2^14, TLC 3-pass 2^15..2^25 (LINES /
    // TILED 3-pass layouts on request), the paper's 5-pass structure (TMA row passes) from 2^26
    // cluster path (one launch, DSMEM exchanges) for 2^15..2^17: 8.3 / 10.0 / 12.5 us vs the
    // three TLC launches' 13.5 / 14.0 / 14.8 us (profiles/r02_small_n.jsonl)
    // (an explicit 3-pass layout or the single-launch TLC option keeps the TLC passes)
    const bool tlc_opts = opt && (opt->layout != 0 || opt->fuse > 0);
    if (passes == 0) passes = (k <= 14) ? 1 : (k <= 17 && !tlc_opts ? 2 : (k <= 25 ? 3 : 5));
    if (opt && opt->layout == 5 && (!opt->passes || opt->passes == 3)) passes = 3;   // TLC ring
    // dense schedule bitstreams only where the 5-pass row kernels read them
    const bool dense_phases = passes == 5 && !(opt && opt->sched_format < 0);
    // geometry of the three phases
    const int64_t lines[3] = {r, c, r};
    const int64_t Ls[3] = {c, r, c};
    const int logLs[3] = {logc, logr, logc};
    for (int f = 0; f < 3; ++f) {
        PhaseGeom& g = P.ph[f];
        g.lines = lines[f];
        g.L = (int32_t)Ls[f];
        g.logL = logLs[f];
        g.E = 2 * g.logL - 5;
        g.epw = 64 / g.E;
        g.w64 = (kW + g.epw - 1) / g.epw;
        // dense for L >= 16384: the schedule-from-global slots (L = 16384) and the half-line
        // ring's staged chunks (L = 32768: five 6.25 KiB chunks in flight instead of four 8 KiB)
        g.dense = dense_phases && (g.logL >= 14 || (opt && opt->sched_format == 2)) ? 1 : 0;
        g.wpl = (int64_t)(g.L / kW) * (g.dense ? g.E : g.w64 * 2);
        g.words = g.lines * g.wpl;
    }
    if (passes == 2) {
        const int st = build_cluster(P, phi, opt, err);
        P.ms_bank = ms_since(t0);
        return st;
    }
    // 5-6. bank-level colouring of every line, packed (W64); not needed by TLC plans
    auto build_line_schedules = [&]() -> int {
        for (int f = 0; f < 3; ++f) {
            PhaseGeom& g = P.ph[f];
            // +4: a dense decode's second load; the device path writes every word, the
            // host path ORs entries into zeroed words
            if (gpu) {
                P.sched[f].resize((size_t)g.words + 4);
                for (int i = 0; i < 4; ++i) P.sched[f][(size_t)g.words + i] = 0u;
            } else {
                P.sched[f].assign((size_t)g.words + 4, 0u);
            }
            const int64_t L = g.L;
            const uint16_t* ph = phi[f].data();
            uint32_t* W = P.sched[f].data();
            auto tph = clk::now();
            if (gpu) {
                // all lines' bank graphs at once on the device (vertex (line, j mod 32) ->
                // (line, Phi(j) mod 32)), colour + W64 packing there
                GpuPlanStats gs;
                const cudaError_t ce = gpu_line_schedules(ph, n, g.logL, g.E, g.epw, g.w64, g.dense, W, &gs);
                if (ce != cudaSuccess) {
                    err = std::string("GPU planner (bank colouring): ") + cudaGetErrorString(ce);
                    return ce == cudaErrorMemoryAllocation ? PERM_ENOMEM : PERM_ECUDA;
                }
                if (std::getenv("PERM_PLANNER_VERBOSE"))
                    std::fprintf(stderr, "[planner] phase %d line schedules (GPU) %.1f ms\n", f, ms_since(tph));
                continue;
            }
#pragma omp parallel
            {
                EulerColourer ec;
                std::vector<uint32_t> U((size_t)L), V((size_t)L), colv((size_t)L);
#pragma omp for schedule(dynamic, 16)
                for (int64_t line = 0; line < g.lines; ++line) {
                    const uint16_t* phl = ph + line * L;
                    uint32_t* col = colv.data();
                    for (int64_t j = 0; j < L; ++j) {
                        U[j] = (uint32_t)(j & 31);
                        V[j] = (uint32_t)(phl[j] & 31);
                    }
                    ec.run(kW, L / kW, L, U.data(), V.data(), col, false);
                    for (int64_t j = 0; j < L; ++j) {
                        const uint64_t sigma = (uint64_t)(j >> 5);
                        const uint64_t entry = (sigma << g.logL) | phl[j];
                        pack_entry(W, g, line, (int64_t)col[j] * kW + (j & 31), entry);
                    }
                }
            }
            if (std::getenv("PERM_PLANNER_VERBOSE"))
                std::fprintf(stderr, "[planner] phase %d line schedules (colour + pack) %.1f ms\n", f, ms_since(tph));
        }
        return PERM_OK;
    };

    // pass structure (chosen above, with the schedule format)
    if (passes == 1 && k > 14) { err = "fused single-CTA pass needs n <= 2^14"; return PERM_EUNSUPPORTED; }
    if (passes != 1 && passes != 3 && passes != 5) { err = "passes must be 0, 1, 3 or 5"; return PERM_EINVAL; }
    P.passes = passes;
    if (passes == 1) {
        P.fused_threads = (int32_t)std::min<int64_t>(512, n / 4);
        P.fused_ept = (int32_t)(n / P.fused_threads);
        P.fused_Ls = (int32_t)(c + 1);   // odd stride: rows AND columns conflict-free (Fig. 4 idea)
        if (r * P.fused_Ls > 65535) { err = "fused tile exceeds 16-bit shared addresses"; return PERM_EUNSUPPORTED; }
        const int bst = build_line_schedules();
        P.ms_bank = ms_since(t0);
        return bst;
    }
    {
        int layout0 = opt ? opt->layout : 0;
        if (passes == 3 && layout0 == 5) {
            const int st = build_tlc_ring(P, phi, opt, err);
            P.ms_bank = ms_since(t0);
            return st;
        }
        if (passes == 3 && (layout0 == 3 || (layout0 == 0 && k >= 15 && k <= 25))) {
            const int st = build_tlc(P, phi, opt, err);
            P.ms_bank = ms_since(t0);
            // one persistent launch when the three passes share the tile size (square view)
            const int fuse = opt ? opt->fuse : 0;
            if (st == PERM_OK && fuse > 0 && P.tp[0].HL == P.tp[1].HL && P.tp[1].HL == P.tp[2].HL &&
                P.tp[0].stages == P.tp[1].stages && P.tp[1].stages == P.tp[2].stages &&
                P.tp[0].bslots == P.tp[1].bslots && P.tp[1].bslots == P.tp[2].bslots &&
                P.tp[0].E == P.tp[1].E && P.tp[1].E == P.tp[2].E)
                P.fused3 = 1;
            return st;
        }
    }
    {
        const int bst = build_line_schedules();
        if (bst != PERM_OK) return bst;
    }
    P.ms_bank = ms_since(t0);
    const int64_t Q = std::min<int64_t>(16384, std::max<int64_t>(2048, pow2_floor(n / 296)));
    auto pick = [&](int idx, int64_t dflt) -> int64_t {
        int64_t v = opt ? (&opt->h1)[idx] : 0;
        return v > 0 ? v : dflt;
    };
    const int stages = (opt && opt->stages > 0) ? opt->stages : 2;
    // bytes of one TMA stage: h lines (stride L + pad) + the tile's packed schedule
    auto stage_bytes = [&](int64_t h, int f, int pad) -> int64_t {
        const PhaseGeom& g = P.ph[f];
        return h * (g.L + pad) * 4 + h * g.wpl * 4;
    };
    constexpr int64_t kSmemBudget = 220 * 1024;
    int layout = opt ? opt->layout : 0;
    if (passes == 3) {
        if (layout == 0) layout = 1;
        if (layout != 1) { err = "layout must be 0, 1 (TILED) or 3 (TLC)"; return PERM_EINVAL; }
    } else {
        layout = 0;
    }
    P.layout = layout;
    if (passes == 3 && layout == 1) {
        int64_t h2 = pick(1, std::min<int64_t>(32, std::max<int64_t>(4, pow2_floor(Q / r))));
        int64_t h1 = pick(0, std::max<int64_t>(1, pow2_floor(Q / c)));
        int64_t h3 = pick(2, h1);
        h2 = std::min(h2, c);
        if (h2 < 4 || h2 > 32 || (h2 & (h2 - 1)) || h1 < 1 || h1 > r || (h1 & (h1 - 1)) ||
            h3 < 1 || h3 > r || (h3 & (h3 - 1))) {
            err = "invalid h1/h2/h3 for the 3-pass layout (h2 in {4,8,16,32}, powers of two)";
            return PERM_EINVAL;
        }
        RowPass& a = P.rp[0];
        a.phase = 0; a.h = (int32_t)h1; a.ctas = r / h1;
        a.in = runs(c, 0, h1 * c);
        a.out = runs(h2, r * h2, h1 * h2);
        RowPass& b = P.rp[1];
        b.phase = 1; b.h = (int32_t)h2; b.ctas = c / h2;
        b.in = cross(r, 0, r * h2);
        b.out = cross(h3, c * h3, h3 * h2);
        RowPass& d = P.rp[2];
        d.phase = 2; d.h = (int32_t)h3; d.ctas = r / h3;
        d.in = runs(h2, h3 * h2, h3 * c);
        d.out = runs(c, 0, h3 * c);
    } else {
        for (int f = 0; f < 3; ++f) {
            const int64_t L = P.ph[f].L, lines_f = P.ph[f].lines;
            // (forced half-line ring: lines of >= 256 words, one line per CTA; a 32-word
            // line would leave a CTA less than one warp)
            const bool force_split = opt && opt->no_tma == -2 && L >= 256;
            int64_t h = force_split ? 1 : pick(f, std::max<int64_t>(1, pow2_floor(Q / L)));
            if (h < 1 || h > lines_f || (h & (h - 1))) { err = "invalid h for the 5-pass layout"; return PERM_EINVAL; }
            RowPass& rp = P.rp[f];
            rp.phase = f; rp.h = (int32_t)h; rp.ctas = lines_f / h;
            rp.in = runs(L, 0, h * L);
            rp.out = runs(L, 0, h * L);
            // TMA pipeline when `stages` tiles (lines + schedule) fit in shared memory
            const bool sched16 = (h * P.ph[f].wpl) % 4 == 0;
            const bool no_tma = opt && opt->no_tma > 0;
            const bool force_sg = opt && opt->no_tma < 0;
            rp.tma = (stages * stage_bytes(h, f, 0) <= kSmemBudget && sched16 && !no_tma && !force_sg) ? 1 : 0;
            rp.stages = rp.tma ? stages : 0;
            // long lines (L >= 16384): the slots hold the data only and the schedule is
            // read from global (L2-prefetched), so 1-3 lines stay in flight per SM
            if (!rp.tma && sched16 && !no_tma && h * L * 4 <= kSmemBudget) {
                rp.tma = 1;
                rp.sg = 1;
                const int64_t fit = kSmemBudget / (h * L * 4);
                rp.stages = (opt && opt->stages > 0) ? opt->stages : (int)std::min<int64_t>(4, fit);
            }
            // one line per slot only (L = 32768): ring of three half-line slots instead
            if (rp.tma && rp.sg && h == 1 && (rp.stages == 1 || force_split) && L >= 256 &&
                3 * (L / 2) * 4 <= kSmemBudget) {
                rp.split = 1;
                rp.stages = 3;
            }
        }
    }
    for (int f = 0; f < 3; ++f) {
        RowPass& rp = P.rp[f];
        const PhaseGeom& g = P.ph[rp.phase];
        if ((int64_t)rp.h * (g.L + 32) > 65535) { err = "tile exceeds 16-bit shared addresses; lower h"; return PERM_EINVAL; }
        choose_threads(rp, g.L);
        if (rp.split) {
            // half-line ring: the schedule streamed through shared-memory chunks by TMA
            // (row_pass_split_stg_kernel, 512 threads) wherever its 64-bit W64 words hold
            // 2 entries or the format is dense and a thread owns 32 or 64 elements (every
            // default plan: L = 32768); otherwise (forced at small L for tests) 512
            // threads re-decode the schedule from global memory in the write hop
            rp.split_keep = 0;
            const int64_t ept512 = (int64_t)rp.h * g.L / 512;
            if ((g.dense || g.w64 == 16) && (ept512 == 32 || ept512 == 64)) {
                rp.split_stg = 1;
                rp.threads = 512;
                rp.ept = (int32_t)ept512;
            } else if ((int64_t)rp.h * g.L >= 8 * 512) {
                rp.threads = 512;
                rp.ept = (int32_t)ept512;
            } else if (rp.ept < 8) {
                rp.ept = 8;
                rp.threads = (int32_t)std::max<int64_t>(32, (int64_t)rp.h * g.L / 8);
            }
        }
        if (rp.tma) {
            // TMA tiles: lines land at 16-byte aligned strides; a CROSS store of h = 8
            // lines needs stride = 4 (mod 8) words to be conflict-free, h = 4 any.
            const int pad = (rp.out.cross && rp.h == 8) ? 4 : 0;
            rp.Ls = g.L + pad;
            rp.conflicts_in = 1;   // bulk copies
            rp.conflicts_out = simulate_conflicts(rp, g, false);
            if ((rp.h * g.wpl) % 4) { err = "TMA tile schedule is not 16-byte sized"; return PERM_EINVAL; }
            const int64_t sb = rp.split ? (int64_t)g.L / 2 * 4
                               : rp.sg ? (int64_t)rp.h * (g.L + pad) * 4 : stage_bytes(rp.h, rp.phase, pad);
            if (rp.stages * sb > kSmemBudget) {
                err = "TMA stages exceed the shared-memory budget; lower h or stages";
                return PERM_EINVAL;
            }
        } else {
            if ((int64_t)rp.h * g.L * 4 > 200 * 1024) { err = "a CTA's lines exceed the shared-memory budget"; return PERM_EINVAL; }
            choose_pad(rp, g);
        }
    }
    return PERM_OK;
}

int build_sharded_plan(const int32_t* p, int64_t n, int32_t eb, int32_t world, int32_t rank,
                       const perm_plan_options* opt, HostPlan& P, std::string& err) {
    if (world < 1 || (world & (world - 1)) || rank < 0 || rank >= world) {
        err = "world must be a power of two and 0 <= rank < world";
        return PERM_EINVAL;
    }
    perm_plan_options o{};
    if (opt) o = *opt;
    o.direct = -1;                      // the shortcut is a single-device kernel
    // TLC form (the column phase's transposes absorbed into the tile-coloured passes, so a
    // step is ONE kernel and the exchange buffers are written / read directly): every rank
    // holds whole tiles of every pass. The send buffers then have exactly the single-GPU
    // X1 / X2 layouts with r -> r/world (X1) and c -> c/world (X2), and a received tile is
    // world segments, one per sender. Otherwise the per-line 5-pass form
    // (R1 + transpose, R2 + transpose, R3), e.g. at 2^26..2^30 or when options ask for it.
    const bool tlc_wanted = (o.passes == 0 || o.passes == 3) && (o.layout == 0 || o.layout == 3) &&
                            o.no_tma == 0 && o.fuse <= 0;
    if (tlc_wanted) {
        const int64_t nw = (eb == 8 ? 2 : 1) * n;
        int kk = 0;
        while ((int64_t(1) << kk) < nw) ++kk;
        if (kk >= 15 && kk <= 25) {
            perm_plan_options ot = o;
            ot.passes = 3;
            ot.layout = 3;
            HostPlan T;
            std::string e2;
            int st = build_host_plan(p, n, eb, &ot, T, e2);
            if (st != PERM_OK) { err = e2; return st; }
            const int64_t r = T.r, c = T.c;
            const int64_t h1 = T.tp[0].h, h2 = T.tp[1].h, h3 = T.tp[2].h;
            if (T.layout == 3 && r % world == 0 && c % world == 0 && (r / world) % h1 == 0 &&
                (c / world) % h2 == 0 && (r / world) % h3 == 0 && r / world >= 32 && c / world >= 32) {
                P = std::move(T);
                P.world = world;
                P.rank = rank;
                P.direct = 0;
                P.p_copy.clear();
                P.r_l = r / world;
                P.c_l = c / world;
                const int64_t Bw = P.r_l * P.c_l;
                const int64_t first[3] = {rank * P.r_l / h1, rank * P.c_l / h2, rank * P.r_l / h3};
                const int64_t count[3] = {P.r_l / h1, P.c_l / h2, P.r_l / h3};
                for (int f = 0; f < 3; ++f) {
                    TlcPass& tp = P.tp[f];
                    U32Buf slice(P.sched[f].begin() + first[f] * tp.tile_words,
                                 P.sched[f].begin() + (first[f] + count[f]) * tp.tile_words);
                    P.sched[f].swap(slice);
                    tp.ntiles = count[f];
                    RowPass& rp = P.rp[f];
                    rp.ctas = count[f];
                    if (f == 0) {
                        tp.segs = 1;
                    } else {
                        tp.segs = world;
                        tp.seg_len = f == 1 ? P.r_l * h2 : P.c_l * h3;
                        tp.seg_stride = Bw;
                    }
                    P.ph[f].lines = count[f] * tp.h;
                }
                return PERM_OK;
            }
        }
    }
    // the global plan with per-line schedules (5-pass geometry: whole lines)
    o.passes = 5;
    o.layout = 0;
    int st = build_host_plan(p, n, eb, &o, P, err);
    if (st != PERM_OK) return st;
    const int64_t r = P.r, c = P.c;
    if (r % world || c % world || r / world < 32 || c / world < 32) {
        err = "row sharding needs r/world >= 32 and c/world >= 32";
        return PERM_EUNSUPPORTED;
    }
    P.world = world;
    P.rank = rank;
    P.direct = 0;                       // the shortcut is a single-device kernel
    P.p_copy.clear();
    P.r_l = r / world;
    P.c_l = c / world;
    const int64_t first[3] = {rank * P.r_l, rank * P.c_l, rank * P.r_l};
    const int64_t count[3] = {P.r_l, P.c_l, P.r_l};
    for (int f = 0; f < 3; ++f) {
        PhaseGeom& g = P.ph[f];
        const int64_t wpl = g.wpl;                                // words per line
        U32Buf slice(P.sched[f].begin() + first[f] * wpl,
                                    P.sched[f].begin() + (first[f] + count[f]) * wpl);
        slice.resize(slice.size() + 4, 0u);      // dense decode's second load stays in bounds
        P.sched[f].swap(slice);
        g.lines = count[f];
        g.words = count[f] * wpl;
        RowPass& rp = P.rp[f];
        if (count[f] % rp.h) rp.h = (int32_t)std::max<int64_t>(1, count[f]);   // degenerate tiny shards
        rp.ctas = count[f] / rp.h;
        rp.in = runs(g.L, 0, (int64_t)rp.h * g.L);
        rp.out = runs(g.L, 0, (int64_t)rp.h * g.L);
        if (f == 0) {
            rp.in_segs = 1;
        } else {
            // each line arrives as `world` segments, one per sender, block-strided
            rp.in_segs = world;
            rp.seg_len = f == 1 ? P.r_l : P.c_l;
            rp.seg_stride = P.r_l * P.c_l;
            // both the TMA pass (one bulk copy per segment) and the plain pass (128-bit
            // loads per segment) gather segmented lines
        }
    }
    return PERM_OK;
}

}  // namespace perm
