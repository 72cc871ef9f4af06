// plan.hpp — host-side plan of the scheduled offline permutation (libperm internals).
//
// PAPER.md §VI-§VII: P is split into three per-line permutations Phi1 (rows),
// Phi2 (columns), Phi3 (rows) of an r x c view (L537-L539, L603-L605), and
// every line's permutation into warp-rounds whose 32 reads and 32 writes hit
// 32 distinct shared-memory banks (L531-L533). This header describes what the
// planner (planner.cpp) produces and the kernels (kernels.cu) consume.
#pragma once

#include <cstdint>
#include <string>
#include <memory>
#include <new>
#include <utility>
#include <vector>

#include "../../include/perm.h"

namespace perm {

constexpr int kW = 32;                 // HMM width w = warp size = banks (L199-L207)

// allocator that default-initialises (no zero fill): large planner arrays that are
// written in full before they are read (zero-filling GBs at n = 2^30 costs seconds)
template <class T>
struct NoInitAlloc : std::allocator<T> {
    template <class U> struct rebind { using other = NoInitAlloc<U>; };
    NoInitAlloc() = default;
    template <class U> NoInitAlloc(const NoInitAlloc<U>&) {}
    template <class U> void construct(U* p) noexcept { ::new ((void*)p) U; }
    template <class U, class... A> void construct(U* p, A&&... a) { ::new ((void*)p) U(std::forward<A>(a)...); }
};
using U16Buf = std::vector<uint16_t, NoInitAlloc<uint16_t>>;
using U32Buf = std::vector<uint32_t, NoInitAlloc<uint32_t>>;

// One phase of row-wise permutations: `lines` independent lines of length L.
// Device schedule ("W64" format): entry = (sigma << logL) | t, E = 2*logL - 5
// bits: the lane reads source position s = 32*sigma + x (bank x) and writes
// destination position t (L519, L533). Entries are packed epw = floor(64/E)
// to a 64-bit word; warp-round (line g, round k) owns W64 = ceil(32/epw)
// consecutive 64-bit words, lane x's entry sits in word x/epw at bit
// E*(x % epw). One 64-bit shared load + one shift decodes it.
struct PhaseGeom {
    int64_t lines = 0;
    int32_t L = 0, logL = 0;
    int32_t E = 0;        // entry bits = logL + (logL - 5)
    int32_t epw = 0;      // entries per 64-bit word
    int32_t w64 = 0;      // 64-bit words per warp-round
    int64_t words = 0;    // 32-bit words: lines * wpl
    // "dense" format (5-pass phases with L >= 16384, where W64 wastes 18-28 of 64
    // bits): warp-round k's 32 entries are one bitstream of E u32 words, lane x's
    // entry at bit x*E (two 32-bit loads + a funnel shift decode it)
    int32_t dense = 0;
    int64_t wpl = 0;      // 32-bit words per line: (L/32) * (dense ? E : 2*w64)
};

// Layout of one row pass of the tiled 3-pass pipeline.
// Element (line l, position pos) of CTA `cta` lives in global memory at
//   RUNS : cta*cta_stride + (pos / w) * strideK + l * w + pos % w
//   CROSS: cta*cta_stride + (pos / blockP) * strideP + (pos % blockP) * h + l
struct IoMode {
    int32_t cross = 0;
    int32_t w = 0;            // RUNS run width (w = L means whole contiguous lines)
    int64_t strideK = 0;      // RUNS
    int32_t blockP = 0;       // CROSS
    int64_t strideP = 0;      // CROSS
    int64_t cta_stride = 0;
};

struct RowPass {
    int32_t phase = 0;        // 0,1,2 -> Phi1, Phi2, Phi3
    int32_t in_segs = 1;      // >1: each input line is in_segs segments (sharded column phase)
    int64_t seg_len = 0, seg_stride = 0;
    int32_t tma = 0;          // 1: persistent TMA-pipelined kernel (contiguous input lines)
    int32_t stages = 0;       // TMA ring depth
    int32_t sg = 0;           // 1 (tma == 1): schedule read from global (L2-prefetched), slots hold data only
    int32_t split = 0;        // 1 (tma == 1, sg, h == 1): ring of three half-line slots (L = 32768)
    int32_t split_keep = 0;   // split: destinations re-decoded in the write hop (the only variant kept)
    int32_t split_stg = 0;    // split: 1 = W64 schedule streamed through smem chunks by a producer warp
    int64_t grid = 0;         // persistent CTAs (set at upload from the occupancy query)
    int32_t h = 0;            // lines per CTA (tile)
    int32_t Ls = 0;           // shared-memory line stride (elements) = L + pad
    int32_t ept = 0;          // elements per thread
    int32_t threads = 0;
    int64_t ctas = 0;
    IoMode in, out;
    int32_t conflicts_in = 1, conflicts_out = 1;   // simulated wavefronts per request
};

// Tile-level-coloured pass (layout TLC): a tile of h lines is loaded by TMA into
// buffer A in its global order, permuted out of place into buffer B laid out
// in the global order of the pass's OUTPUT, and stored by TMA. The bank graph
// of the whole tile (edge (src mod 32, dst mod 32) per element, src/dst = word
// offsets in A/B) is (HL/32)-regular; its König colouring gives warp-rounds
// that read 32 distinct banks of A and write 32 distinct banks of B, whatever
// the two layouts are. Entry (lane x = src bank, round q) = ((src >> 5) <<
// logHL) | dst, E = 2*logHL - 5 bits. Permuter warp pw owns rounds
// [pw*ept, (pw+1)*ept); each lane keeps its ept entries as one bitstream of
// nwords u32 words; word w of lane x of (tile T, warp pw) is stored at
// ((T*NW + pw)*nwords + w)*32 + x (coalesced loads).
constexpr int kTlcPerm = 512;           // permuter threads per CTA

// Destination of a TLC entry. An element never leaves its line in a row-wise
// permutation (L517), so the line's index inside the tile is a function of the
// source offset; the entry keeps only t = the destination position in the line
// (log2 L bits) and the kernel rebuilds
//   dst = ((t >> s1) << s2) | (((src >> s4) & m2) << s3) | (t & m1),
// E = (logHL - 5) + lt bits ("compact"; 19 at n = 2^22 vs 21). The full format
// (lt = logHL, dst = t: s1 = s2 = s3 = s4 = m1 = m2 = 0) is kept for entry
// widths without a compiled kernel (tlc_compact_supported).
struct TlcDecode {
    int32_t lt = 0;
    int32_t s1 = 0, s2 = 0, s3 = 0, s4 = 0;
    uint32_t m1 = 0, m2 = 0;
};
inline uint32_t tlc_dst(const TlcDecode& d, uint32_t t, uint32_t src) {
    return ((t >> d.s1) << d.s2) | (((src >> d.s4) & d.m2) << d.s3) | (t & d.m1);
}
// (elements per permuter thread, compact entry bits) pairs with a compiled kernel
inline bool tlc_compact_supported(int ept, int E) {
    return (ept == 16 && E >= 15 && E <= 20) || (ept == 32 && (E == 21 || E == 22));
}

struct TlcPass {
    int32_t h = 0;            // lines per tile
    int32_t HL = 0, logHL = 0;
    int32_t E = 0;
    int32_t ept = 0;          // HL / kTlcPerm
    int32_t nwords = 0;       // ceil(ept * E / 32)
    int64_t ntiles = 0;
    int64_t tile_words = 0;   // (kTlcPerm / 32) * nwords * 32
    int32_t out_kind = 0;     // 0: rows (1-D bulk store); 1: X1 / 2: X2 2-D tensor store (64-byte box rows)
    TlcDecode dec;            // entry -> destination offset (compact or full format)
    int32_t stages = 0;       // A slots (TMA loads in flight); B slots = bslots
    int32_t bslots = 0;       // B slots (permuted tiles waiting for / under their TMA store)
    int64_t grid = 0;         // persistent CTAs (set at upload)
    // row-sharded TLC: a tile arrives as `segs` segments of seg_len words, one
    // per sender, at in + s*seg_stride + t*seg_len (segs = 1: the tile is in[t*HL, +HL))
    int32_t segs = 1;
    int64_t seg_len = 0, seg_stride = 0;
};

struct HostPlan {
    int64_t n = 0;             // words permuted (2 * user_n for 8-byte elements)
    int32_t eb = 4;            // word size used by the kernels (always 4)
    int32_t user_eb = 4;       // element size of the caller (4 or 8)
    int64_t user_n = 0;        // elements of the caller
    int32_t k = 0;             // log2 n
    int64_t r = 0, c = 0;      // view
    int32_t passes = 0;        // 1, 3, 5; 2 = cluster path (one launch, DSMEM exchanges)
    int32_t cluster = 0;       // cluster path: thread blocks in the cluster (C)
    int32_t layout = 0;        // 3-pass intermediates: 1 tiled, 2 lines, 3 TLC; 4 = cluster path
    int32_t fused3 = 0;        // LINES layout, square view: all three passes in one launch
    TlcPass tp[3];             // layout TLC (3): the three passes
    // row-sharded plans: this rank owns rows [rank*r_l, +r_l) of a and b,
    // and columns [rank*c_l, +c_l) in the column phase; schedules are sliced to those lines
    int32_t world = 1, rank = 0;
    // low-distribution shortcut: D_w(P) <= 2n/w -> the D-designated kernel (coalesced)
    int64_t distribution = 0;
    int32_t direct = 0;
    std::vector<int32_t> p_copy;   // uploaded for the direct kernel
    int64_t r_l = 0, c_l = 0;
    int64_t fused3_grid = 0;   // one CTA per SM (set at upload)
    PhaseGeom ph[3];
    RowPass rp[3];
    int32_t fused_ept = 0, fused_threads = 0, fused_Ls = 0;
    std::vector<uint16_t> kappa;
    U32Buf sched[3];
    double ms_colour = 0, ms_bank = 0;
    int32_t threads_used = 1;
    int32_t gpu_planner = 0;   // 1: colourings ran on the device (gplan.cu)
};

// Builds everything host-side. Returns PERM_OK or a perm_status, with `err` set.
int build_host_plan(const int32_t* p, int64_t n, int32_t eb, const perm_plan_options* opt,
                    HostPlan& out, std::string& err);

// Row-sharded plan for `rank` of `world` (world a power of two dividing r and c):
// the global colouring, then this rank's slices of the three phase schedules.
int build_sharded_plan(const int32_t* p, int64_t n, int32_t eb, int32_t world, int32_t rank,
                       const perm_plan_options* opt, HostPlan& out, std::string& err);

// Colour a d-regular bipartite multigraph (d a power of two) with d colours by
// recursive Euler splitting. U[e], V[e] < nodes, E = nodes * d edges.
void euler_split_colour(int64_t nodes, int64_t d, int64_t E, const uint32_t* U,
                        const uint32_t* V, uint32_t* colour, bool parallel);

// Position of the entry of (line, slot q = round*32 + lane) in a W64 phase.
inline void entry_pos(const PhaseGeom& g, int64_t line, int64_t q, int64_t& word64, int& bit) {
    const int64_t round = q >> 5, lane = q & 31;
    word64 = (line * (g.L >> 5) + round) * g.w64 + lane / g.epw;
    bit = (int)(g.E * (lane % g.epw));
}

// 32-bit word index and bit offset (< 32) of entry (line, slot q) in either format
inline void entry_pos32(const PhaseGeom& g, int64_t line, int64_t q, int64_t& wi, int& b) {
    if (g.dense) {
        const int64_t round = q >> 5, lane = q & 31;
        const int64_t bit = lane * g.E;
        wi = line * g.wpl + round * g.E + (bit >> 5);
        b = (int)(bit & 31);
    } else {
        int64_t w64;
        int bit;
        entry_pos(g, line, q, w64, bit);
        wi = 2 * w64 + (bit >> 5);
        b = bit & 31;
    }
}

inline void pack_entry(uint32_t* words, const PhaseGeom& g, int64_t line, int64_t q, uint64_t entry) {
    int64_t wi;
    int b;
    entry_pos32(g, line, q, wi, b);
    const uint64_t sh = entry << b;
    words[wi] |= (uint32_t)sh;
    if (b + g.E > 32) words[wi + 1] |= (uint32_t)(sh >> 32);
}

inline uint32_t unpack_entry(const U32Buf& words, const PhaseGeom& g,
                             int64_t line, int64_t q) {
    int64_t wi;
    int b;
    entry_pos32(g, line, q, wi, b);
    uint64_t v = words[wi];
    if (b + g.E > 32) v |= (uint64_t)words[wi + 1] << 32;
    return (uint32_t)((v >> b) & ((1ull << g.E) - 1));
}

// Entry of (tile T, warp-round q, lane x) of a TLC pass.
inline uint32_t tlc_entry(const U32Buf& words, const TlcPass& tp, int64_t T,
                          int64_t q, int64_t x) {
    const int64_t pw = q / tp.ept, m = q % tp.ept;
    const int64_t bit = m * tp.E, w = bit >> 5, off = bit & 31;
    const uint32_t* base = words.data() + T * tp.tile_words + pw * tp.nwords * 32 + x;
    uint64_t v = base[w * 32];
    if (off + tp.E > 32) v |= (uint64_t)base[(w + 1) * 32] << 32;
    return (uint32_t)((v >> off) & ((1ull << tp.E) - 1));
}

// Simulated shared-memory wavefronts per warp request of a pass's load/store
// loops (1 = conflict-free). Mirrors the index math in kernels.cu.
int simulate_conflicts(const RowPass& rp, const PhaseGeom& g, bool input_side);

}  // namespace perm
