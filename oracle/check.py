"""Invariants every valid scheduled-permutation plan satisfies. ORACLE — test infrastructure only.

A plan is (kappa, {(sigma_phi, t_phi)}_{phi=1,2,3}) on an r x c view. The
checker rebuilds Phi1..Phi3 from kappa and p itself (it never trusts a
plan's own phase arrays) and verifies, vectorised so it scales to any n:

 (i)   kappa restricted to each row is a bijection onto [0, c)        (L537 (1))
 (ii)  within each colour class the destination rows are distinct      (L537 (2))
 (iii) every Phi restricted to every line is a bijection               (L517)
 (iv)  routing x through Phi1, Phi2, Phi3 lands at P(x)                (L539)
 (v)   t = Phi(s) slot by slot, with s = w*sigma + lane                (L519)
 (vi)  every warp-round reads w distinct banks and writes w distinct
       banks                                                           (L531-L533, L213)
 (vii) the s of each line cover [0, L) exactly once                   (L521-L525)
"""
from __future__ import annotations

import numpy as np


def phases_from_kappa(p: np.ndarray, kappa: np.ndarray, rows: int, cols: int):
    """Phi1 (r,c), Phi2 (c,r), Phi3 (r,c) from kappa and P (L537-L539), vectorised."""
    p = np.asarray(p, dtype=np.int64)
    kappa = np.asarray(kappa, dtype=np.int64)
    n = rows * cols
    x = np.arange(n, dtype=np.int64)
    src_row = x // cols
    dest_row, dest_col = p // cols, p % cols
    phi1 = kappa.reshape(rows, cols).copy()
    phi2 = np.full((cols, rows), -1, dtype=np.int64)
    phi3 = np.full((rows, cols), -1, dtype=np.int64)
    phi2[kappa, src_row] = dest_row
    phi3[dest_row, kappa] = dest_col
    return phi1, phi2, phi3


def _rows_are_perms(m: np.ndarray) -> bool:
    L = m.shape[1]
    if m.min() < 0 or m.max() >= L:
        return False
    s = np.sort(m, axis=1)
    return bool(np.all(s == np.arange(L, dtype=s.dtype)[None, :]))


def _rounds_distinct(v: np.ndarray, w: int) -> bool:
    """v shape (lines, L): every group of w consecutive slots has distinct v mod w."""
    lines, L = v.shape
    b = np.sort((v % w).reshape(lines, L // w, w), axis=2)
    return bool(np.all(b == np.arange(w)[None, None, :]))


def check_plan(p, kappa, sched, rows: int, cols: int, w: int) -> dict:
    """Return {invariant: bool}. ``sched`` = [(sigma1, t1), (sigma2, t2), (sigma3, t3)]
    with shapes (r, c), (c, r), (r, c) in logical [line][slot] order."""
    p = np.asarray(p, dtype=np.int64)
    kappa = np.asarray(kappa, dtype=np.int64)
    n = rows * cols
    res = {}
    res["shape"] = (p.size == n and kappa.size == n)
    if not res["shape"]:
        return res
    # (i)
    res["i_row_colours_bijective"] = _rows_are_perms(kappa.reshape(rows, cols))
    # (ii)
    key = kappa * rows + p // cols
    res["ii_colour_dest_rows_distinct"] = bool(
        kappa.min() >= 0 and kappa.max() < cols and np.unique(key).size == n)
    if not (res["i_row_colours_bijective"] and res["ii_colour_dest_rows_distinct"]):
        return res
    phis = phases_from_kappa(p, kappa, rows, cols)
    # (iii)
    res["iii_phases_bijective"] = all(_rows_are_perms(ph) for ph in phis)
    # (iv)
    x = np.arange(n, dtype=np.int64)
    i, j = x // cols, x % cols
    k = phis[0][i, j]
    row2 = phis[1][k, i]
    col3 = phis[2][row2, k]
    res["iv_composition_is_P"] = bool(np.all(row2 * cols + col3 == p))
    ok_v = ok_vi = ok_vii = True
    for phi, (sig, t) in zip(phis, sched):
        sig = np.asarray(sig, dtype=np.int64)
        t = np.asarray(t, dtype=np.int64)
        lines, L = phi.shape
        if sig.shape != (lines, L) or t.shape != (lines, L):
            ok_v = ok_vi = ok_vii = False
            continue
        lane = np.arange(L, dtype=np.int64)[None, :] % w
        s = w * sig + lane
        if s.min() < 0 or s.max() >= L:
            ok_v = ok_vi = ok_vii = False
            continue
        ok_vii &= _rows_are_perms(s)
        ok_v &= bool(np.all(np.take_along_axis(phi, s, axis=1) == t))
        ok_vi &= _rounds_distinct(s, w) and _rounds_distinct(t, w)
    res["v_t_equals_phi_of_s"] = ok_v
    res["vi_rounds_conflict_free"] = ok_vi
    res["vii_sources_cover_line"] = ok_vii
    return res


def assert_plan(p, kappa, sched, rows, cols, w):
    res = check_plan(p, kappa, sched, rows, cols, w)
    bad = [k for k, v in res.items() if not v]
    expected = {"shape", "i_row_colours_bijective", "ii_colour_dest_rows_distinct",
                "iii_phases_bijective", "iv_composition_is_P", "v_t_equals_phi_of_s",
                "vi_rounds_conflict_free", "vii_sources_cover_line"}
    missing = expected - set(res)
    if bad or missing:
        raise AssertionError(f"plan invariants failed: {bad} missing: {sorted(missing)}")
    return res


# ---------------------------------------------------------------- tile-level coloured plans
#
# DESIGN.md §5 "TLC": each of the three row-wise permutations runs on tiles of h
# lines. A tile is read from global memory in its stored order into buffer A and
# written in the stored order of the pass's output into buffer B; a plan entry
# (tile T, warp-round q, lane x) is (src offset in A, dst offset in B). The
# layouts (restated here from DESIGN.md, not imported from the product):
#   X1[((K*(r/h1) + I)*h1 + i_in)*h2 + k_in]        (K = k div h2, I = i div h1)
#   X2[((I'*(c/h2) + K)*h3 + i_in')*h2 + k_in]
#   pass 1, tile I : A = rows I*h1.. of a (i_in*c + j);       B = [K][i_in][k_in]
#   pass 2, tile K : A = X1 block K   ([i][k_in]);            B = [I'][i_in'][k_in]
#   pass 3, tile I': A = X2 block I'  ([K][i_in'][k_in]);     B = rows of b (i_in'*c + k')
# The checker maps every src back to its element, routes the element with the
# Phi it recomputes from kappa and P, and requires: dst = the layout position of
# the routed element (i.e. the pass implements Phi), every src and every dst of
# a tile used once, lane = src mod w, and every round touching w distinct banks
# in A and in B (L531-L533 generalised from a line to a tile).

def check_tlc(p, kappa, sched, rows: int, cols: int, h, w: int = 32) -> dict:
    p = np.asarray(p, dtype=np.int64)
    kappa = np.asarray(kappa, dtype=np.int64)
    r, c = rows, cols
    h1, h2, h3 = h
    n = r * c
    res = {}
    res["i_row_colours_bijective"] = _rows_are_perms(kappa.reshape(r, c))
    key = kappa * r + p // c
    res["ii_colour_dest_rows_distinct"] = bool(np.unique(key).size == n)
    if not (res["i_row_colours_bijective"] and res["ii_colour_dest_rows_distinct"]):
        return res
    phi1, phi2, phi3 = phases_from_kappa(p, kappa, r, c)
    ok_map = ok_cover = ok_banks = ok_lane = True
    for f, (HL, lines, hh) in enumerate(((h1 * c, r, h1), (r * h2, c, h2), (h3 * c, r, h3))):
        e = np.asarray(sched[f], dtype=np.int64).reshape(lines // hh, HL)
        src, dst = e >> 16, e & 0xFFFF
        T = np.arange(lines // hh, dtype=np.int64)[:, None]
        lane = (np.arange(HL, dtype=np.int64) % w)[None, :]
        ok_lane &= bool(np.all(src % w == lane))
        ok_cover &= _rows_are_perms(src) and _rows_are_perms(dst)
        ok_banks &= _rounds_distinct(src, w) and _rounds_distinct(dst, w)
        if f == 0:
            i = T * h1 + src // c
            j = src % c
            k = phi1[i, j]
            want = ((k // h2) * h1 + (i - T * h1)) * h2 + k % h2
        elif f == 1:
            i = src // h2
            k = T * h2 + src % h2
            ip = phi2[k, i]
            want = ip * h2 + (k - T * h2)
        else:
            K, rem = src // (h3 * h2), src % (h3 * h2)
            i_in, k_in = rem // h2, rem % h2
            k = K * h2 + k_in
            ip = T * h3 + i_in
            want = i_in * c + phi3[ip, k]
        ok_map &= bool(np.all(dst == want))
    res["iii_phases_bijective"] = all(_rows_are_perms(ph) for ph in (phi1, phi2, phi3))
    x = np.arange(n, dtype=np.int64)
    i, j = x // c, x % c
    k = phi1[i, j]
    row2 = phi2[k, i]
    res["iv_composition_is_P"] = bool(np.all(row2 * c + phi3[row2, k] == p))
    res["v_tiles_implement_phi"] = ok_map
    res["vi_rounds_conflict_free_A_and_B"] = ok_banks
    res["vii_sources_and_dests_cover_tile"] = ok_cover
    res["viii_lane_is_source_bank"] = ok_lane
    return res


# ---------------------------------------------------------------- cluster plans
#
# DESIGN.md §5 "cluster path" (restated, not imported): C thread blocks of one cluster
# hold the whole array; r_l = r/C, c_l = c/C, Bw = r_l*c_l. Block g's phase-1 input is
# rows [g*r_l, ...) of a (row-major); its phase-1 output is C send blocks, element
# (i, k) in block k div c_l at [k mod c_l][i mod r_l]; the exchange delivers send block
# q of block g to block q at [g*Bw, (g+1)*Bw). Phase 2 output: send block i' div r_l at
# [i' mod r_l][k mod c_l]; phase 3 output: block m's rows of b, row-major. The checker
# derives every element from its SOURCE offset (the input side of each phase), routes
# it with the Phi it recomputes, and compares with the destination offset.

def check_cluster(p, kappa, sched, rows: int, cols: int, C: int, w: int = 32) -> dict:
    p = np.asarray(p, dtype=np.int64)
    kappa = np.asarray(kappa, dtype=np.int64)
    r, c = rows, cols
    n = r * c
    rl, cl, S = r // C, c // C, n // C
    Bw = rl * cl
    res = {}
    res["i_row_colours_bijective"] = _rows_are_perms(kappa.reshape(r, c))
    res["ii_colour_dest_rows_distinct"] = bool(np.unique(kappa * r + p // c).size == n)
    if not (res["i_row_colours_bijective"] and res["ii_colour_dest_rows_distinct"]):
        return res
    phi1, phi2, phi3 = phases_from_kappa(p, kappa, r, c)
    ok_map = ok_cover = ok_banks = ok_lane = True
    g = np.arange(C, dtype=np.int64)[:, None]
    for f in range(3):
        e = np.asarray(sched[f], dtype=np.int64).reshape(C, S)
        src, dst = e >> 16, e & 0xFFFF
        lane = (np.arange(S, dtype=np.int64) % w)[None, :]
        ok_lane &= bool(np.all(src % w == lane))
        ok_cover &= _rows_are_perms(src) and _rows_are_perms(dst)
        ok_banks &= _rounds_distinct(src, w) and _rounds_distinct(dst, w)
        if f == 0:
            i = g * rl + src // c
            k = phi1[i, src % c]
            want = (k // cl) * Bw + (k % cl) * rl + i % rl
        elif f == 1:
            sender, rem = src // Bw, src % Bw
            k_in, i_l = rem // rl, rem % rl
            ip = phi2[g * cl + k_in, sender * rl + i_l]
            want = (ip // rl) * Bw + (ip % rl) * cl + k_in
        else:
            sender, rem = src // Bw, src % Bw
            i_l, k_in = rem // cl, rem % cl
            kp = phi3[g * rl + i_l, sender * cl + k_in]
            want = i_l * c + kp
        ok_map &= bool(np.all(dst == want))
    x = np.arange(n, dtype=np.int64)
    i, j = x // c, x % c
    k = phi1[i, j]
    row2 = phi2[k, i]
    res["iii_phases_bijective"] = all(_rows_are_perms(ph) for ph in (phi1, phi2, phi3))
    res["iv_composition_is_P"] = bool(np.all(row2 * c + phi3[row2, k] == p))
    res["v_blocks_implement_phi"] = ok_map
    res["vi_rounds_conflict_free_A_and_B"] = ok_banks
    res["vii_sources_and_dests_cover_block"] = ok_cover
    res["viii_lane_is_source_bank"] = ok_lane
    return res
