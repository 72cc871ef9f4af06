"""Tiled forms of the scheduled permutation, built and executed by the oracle. ORACLE —
test infrastructure only.

The product runs the row-wise permutations of Thm 9 (L537-L539) on TILES rather
than on single lines, and colours each tile's bank graph between the tile's input
order and its output order (L531-L533 generalised from a line to a tile: the
bipartite graph with one edge (src mod w, dst mod w) per element is (HL/w)-regular
because both buffers are dense, so König (Thm 6) gives HL/w warp-rounds that
read w distinct banks and write w distinct banks). Two tiled forms exist; their
storage layouts are restated here from DESIGN.md §5 (never imported from the
product), and this module builds plans for them with the oracle's own colourings
(konig.py, alternating paths) and executes plans -- the oracle's or the product's
exported ones -- on numpy arrays.

TLC (three passes through global memory), tiles of h1 / h2 / h3 lines:
  pass 1: tile T = rows [T*h1, (T+1)*h1) of a (contiguous). Its output buffer B is
          c/h2 chunks of cw = h1*h2 words; chunk m holds columns [m*h2, (m+1)*h2)
          of the tile's rows as [row in tile][column in chunk]. Chunk m of tile T is
          stored at X1[m*(r*h2) + T*cw ...].
  pass 2: tile K = X1[K*r*h2 : (K+1)*r*h2] (columns [K*h2, (K+1)*h2) of all rows, as
          [row][column in block]). B = r/h3 chunks of cw = h3*h2 words; chunk m
          holds rows [m*h3, (m+1)*h3) as [row in chunk][column in block], stored at
          X2[m*(c*h3) + K*cw ...].
  pass 3: tile I' = X2[I'*c*h3 : (I'+1)*c*h3]; B = rows [I'*h3, (I'+1)*h3) of b,
          row-major, stored at b[I'*h3*c ...] (one chunk).

CLUSTER (one launch; the whole array in the shared memory of C thread blocks; the
column phase's two transposes, Lemma 8, become two all-to-all exchanges of
uniform blocks between the blocks, like the row-sharded multi-GPU form):
  r_l = r/C, c_l = c/C, S = n/C, Bw = r_l*c_l. Block g owns rows [g*r_l, (g+1)*r_l)
  in phases 1 and 3 and columns [g*c_l, (g+1)*c_l) in phase 2.
  phase 1 (block g): A = a[g*S : (g+1)*S]; B = C send blocks; element (row i, column
          k) after the phase sits in send block k div c_l at [k mod c_l][i mod r_l].
  exchange: block g's send block q -> block q's receive buffer at [g*Bw : (g+1)*Bw].
  phase 2 (block q): A = receive buffer; element (row i', column k) after the phase
          sits in send block i' div r_l at [i' mod r_l][k mod c_l].
  exchange (as above).
  phase 3 (block m): A = receive buffer; B = rows of b owned by m, row-major; stored
          at b[m*S : (m+1)*S].

Plans are lists (one per pass / phase) of flat uint32 arrays: entry
[tile * HL + round * w + lane] = (src << 16) | dst, src / dst = word offsets in the
tile's A / B buffers, lane = src mod w (reading #8 of DESIGN.md).
"""
from __future__ import annotations

import numpy as np

from .konig import edge_colour
from .planner import phase_permutations, row_colouring


# ------------------------------------------------------------------ shared helpers

def _tile_schedule(src: np.ndarray, dst: np.ndarray, w: int) -> np.ndarray:
    """Colour one tile's bank graph (edge (src mod w, dst mod w) per element) with the
    oracle's König colouring; colour k = warp-round k, lane = source bank."""
    HL = src.size
    edges = [(int(s) % w, int(d) % w) for s, d in zip(src, dst)]
    colour = edge_colour(w, w, edges, HL // w)
    out = np.zeros(HL, dtype=np.uint32)
    for e in range(HL):
        slot = colour[e] * w + int(src[e]) % w
        out[slot] = (int(src[e]) << 16) | int(dst[e])
    return out


def _run_tile(A: np.ndarray, entries: np.ndarray, w: int, stats: dict) -> np.ndarray:
    """B[dst] = A[src] round by round; counts rounds and conflict-free rounds."""
    src = (entries >> 16).astype(np.int64)
    dst = (entries & 0xFFFF).astype(np.int64)
    B = np.empty_like(A)
    for q in range(src.size // w):
        s = src[q * w:(q + 1) * w]
        d = dst[q * w:(q + 1) * w]
        stats["rounds"] += 1
        if len(set((s % w).tolist())) == w and len(set((d % w).tolist())) == w:
            stats["conflict_free"] += 1
        B[d] = A[s]
    return B


# ------------------------------------------------------------------ TLC form

def tlc_geometry(rows: int, cols: int, h):
    """Per pass: (tiles, HL, chunk words cw, chunk stride in the output)."""
    r, c = rows, cols
    h1, h2, h3 = h
    return [(r // h1, h1 * c, h1 * h2, r * h2),
            (c // h2, r * h2, h3 * h2, c * h3),
            (r // h3, h3 * c, h3 * c, h3 * c)]


def tlc_plan(p, rows: int, cols: int, h, w: int = 32):
    """(kappa, [sched1, sched2, sched3]) of the TLC form, built by following every
    element through the three passes (labels), with the oracle's own colourings."""
    p = np.asarray(p, dtype=np.int64)
    r, c = rows, cols
    h1, h2, h3 = h
    n = r * c
    kappa = row_colouring(p, r, c)
    phi1, phi2, phi3 = phase_permutations(p, kappa, r, c)
    geo = tlc_geometry(r, c, h)
    # where[x] = (row, column) of element x in the logical r x c matrix before each pass
    row = np.arange(n) // c
    col = np.arange(n) % c
    store = np.arange(n)                  # store[pos] = element at storage position pos
    scheds = []
    for f in range(3):
        ntiles, HL, cw, cstride = geo[f]
        sched = np.zeros(ntiles * HL, dtype=np.uint32)
        nxt = np.empty(n, dtype=np.int64)
        nrow, ncol = row.copy(), col.copy()
        for T in range(ntiles):
            elems = store[T * HL:(T + 1) * HL]
            src = np.arange(HL)
            dst = np.empty(HL, dtype=np.int64)
            for s, x in enumerate(elems):
                i, k = int(row[x]), int(col[x])
                if f == 0:                       # row-wise: column k -> phi1
                    k = int(phi1[i, k])
                    dst[s] = (k // h2) * cw + (i - T * h1) * h2 + k % h2
                elif f == 1:                     # column-wise: row i -> phi2
                    i = int(phi2[k, i])
                    dst[s] = (i // h3) * cw + (i % h3) * h2 + (k - T * h2)
                else:                            # row-wise: column k -> phi3
                    k = int(phi3[i, k])
                    dst[s] = (i - T * h3) * c + k
                nrow[x], ncol[x] = i, k
            sched[T * HL:(T + 1) * HL] = _tile_schedule(src, dst, w)
            B = np.empty(HL, dtype=np.int64)
            B[dst] = elems
            for m in range(HL // cw):
                nxt[m * cstride + T * cw:m * cstride + (T + 1) * cw] = B[m * cw:(m + 1) * cw]
        store, row, col = nxt, nrow, ncol
        scheds.append(sched)
    return kappa, scheds


def tlc_apply(a: np.ndarray, scheds, rows: int, cols: int, h, w: int = 32):
    """Execute a TLC plan: per pass, per tile, A = the tile's input range, B[dst] = A[src]
    round by round, then B's chunks to their output positions. Returns (b, stats)."""
    X = np.ascontiguousarray(a).copy()
    stats = {"rounds": 0, "conflict_free": 0}
    for f, (ntiles, HL, cw, cstride) in enumerate(tlc_geometry(rows, cols, h)):
        e = np.asarray(scheds[f], dtype=np.uint32).reshape(ntiles, HL)
        Y = np.empty_like(X)
        for T in range(ntiles):
            B = _run_tile(X[T * HL:(T + 1) * HL], e[T], w, stats)
            for m in range(HL // cw):
                Y[m * cstride + T * cw:m * cstride + (T + 1) * cw] = B[m * cw:(m + 1) * cw]
        X = Y
    return X, stats


# ------------------------------------------------------------------ cluster form

def cluster_plan(p, rows: int, cols: int, C: int, w: int = 32):
    """(kappa, [sched1, sched2, sched3]) of the CLUSTER form: per phase, C tiles (one per
    thread block) of S = n/C entries, built by following the elements, oracle colourings."""
    p = np.asarray(p, dtype=np.int64)
    r, c = rows, cols
    n = r * c
    rl, cl, S = r // C, c // C, n // C
    Bw = rl * cl
    kappa = row_colouring(p, r, c)
    phi1, phi2, phi3 = phase_permutations(p, kappa, r, c)
    row = np.arange(n) // c
    col = np.arange(n) % c
    bufs = [np.arange(g * S, (g + 1) * S) for g in range(C)]   # element in each block's A
    scheds = []
    for f in range(3):
        sched = np.zeros(C * S, dtype=np.uint32)
        outs = []
        for g in range(C):
            elems = bufs[g]
            dst = np.empty(S, dtype=np.int64)
            for s, x in enumerate(elems):
                i, k = int(row[x]), int(col[x])
                if f == 0:
                    k = int(phi1[i, k])
                    dst[s] = (k // cl) * Bw + (k % cl) * rl + i % rl
                elif f == 1:
                    i = int(phi2[k, i])
                    dst[s] = (i // rl) * Bw + (i % rl) * cl + k % cl
                else:
                    k = int(phi3[i, k])
                    dst[s] = (i - g * rl) * c + k
                row[x], col[x] = i, k
            sched[g * S:(g + 1) * S] = _tile_schedule(np.arange(S), dst, w)
            B = np.empty(S, dtype=np.int64)
            B[dst] = elems
            outs.append(B)
        if f < 2:      # exchange: block g's send block q -> block q's A at [g*Bw, (g+1)*Bw)
            bufs = [np.concatenate([outs[g][q * Bw:(q + 1) * Bw] for g in range(C)]) for q in range(C)]
        scheds.append(sched)
    return kappa, scheds


def cluster_apply(a: np.ndarray, scheds, rows: int, cols: int, C: int, w: int = 32):
    """Execute a CLUSTER plan block by block with the two block exchanges. (b, stats)."""
    n = rows * cols
    S, Bw = n // C, (rows // C) * (cols // C)
    X = np.ascontiguousarray(a)
    bufs = [X[g * S:(g + 1) * S].copy() for g in range(C)]
    stats = {"rounds": 0, "conflict_free": 0}
    for f in range(3):
        e = np.asarray(scheds[f], dtype=np.uint32).reshape(C, S)
        outs = [_run_tile(bufs[g], e[g], w, stats) for g in range(C)]
        if f < 2:
            bufs = [np.concatenate([outs[g][q * Bw:(q + 1) * Bw] for g in range(C)]) for q in range(C)]
        else:
            bufs = outs
    return np.concatenate(bufs), stats
