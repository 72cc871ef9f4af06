"""Reference planner for the scheduled permutation. ORACLE — test infrastructure only.

Follows PAPER.md in its own order and notation:

§VII (L603-L605, L537-L539). View a and b as r x c matrices (L603: "not
restricted to a square matrix"); element x = i*c + j of a is in row i and
must reach b[P(x)], row P(x) div c, column P(x) mod c. Draw the bipartite
multigraph with U = rows of a, V = rows of b and one edge
(u_i, v_{P(x) div c}) per element: it is c-regular, so by König (Thm 6)
it is c-edge-colourable. With colour kappa(x):
  (1) numbers in the same row have different colours,
  (2) numbers with the same colour have different destination rows.
Step 1 (row-wise): the number with colour k moves to column k.
Step 2 (column-wise): each number moves to its destination row.
Step 3 (row-wise): each number moves to its destination column.

§VI (L517-L533). A row-wise permutation moves b[i][P_i(j)] <- a[i][j]. It
runs as B_i[t_i(j)] <- A_i[s_i(j)] with t_i(j) = P_i(s_i(j)) (L519). The
bank-level graph has U = banks of A_i, V = banks of B_i and one edge
(u_{j mod w}, v_{P_i(j) mod w}) per j; it is (L/w)-regular, so it has an
(L/w)-edge-colouring. r_k(x) is the source index of the colour-k edge that
leaves bank x; s_i(k*w + x) = r_k(x) and t_i(k*w + x) = P_i(r_k(x)) (L531-L533),
so warp k reads w distinct banks and writes w distinct banks.

The schedule is returned as (sigma, t) with s = w*sigma + lane (reading #8 in
DESIGN.md: lane x takes the source in bank x, so s mod w = x).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .konig import edge_colour


@dataclass
class Plan:
    n: int
    rows: int
    cols: int
    w: int
    kappa: np.ndarray                      # kappa[x], colour of element x (row level)
    phi: list = field(default_factory=list)    # [phi1 (r,c), phi2 (c,r), phi3 (r,c)]
    sigma: list = field(default_factory=list)  # per phase: (lines, L) row-in-bank of s
    t: list = field(default_factory=list)      # per phase: (lines, L) destination index


def default_view(n: int) -> tuple[int, int]:
    m = n.bit_length() - 1
    if (1 << m) == n:
        return 1 << (m // 2), 1 << (m - m // 2)
    r = int(round(n ** 0.5))
    if r * r != n:
        raise ValueError("n must be a power of two or a perfect square")
    return r, r


def row_colouring(p: np.ndarray, rows: int, cols: int) -> np.ndarray:
    """kappa: a proper cols-edge-colouring of the row-level multigraph (L603-L605)."""
    n = rows * cols
    edges = [(x // cols, int(p[x]) // cols) for x in range(n)]
    return np.asarray(edge_colour(rows, rows, edges, cols), dtype=np.int64)


def phase_permutations(p: np.ndarray, kappa: np.ndarray, rows: int, cols: int):
    """Phi1, Phi2, Phi3 as per-line permutations (L537-L539).

    phi1[i][j]  = kappa(i*c + j)          step 1 within row i
    phi2[k][i]  = P(x) div c              step 2 within column k, x = the element
                                          of row i with colour k
    phi3[i'][k] = P(x) mod c              step 3 within row i', x = the element
                                          that step 2 brought to (i', k)
    """
    p = np.asarray(p, dtype=np.int64)
    n = rows * cols
    phi1 = np.empty((rows, cols), dtype=np.int64)
    phi2 = np.full((cols, rows), -1, dtype=np.int64)
    phi3 = np.full((rows, cols), -1, dtype=np.int64)
    for x in range(n):
        i, j = divmod(x, cols)
        k = int(kappa[x])
        dest_row, dest_col = divmod(int(p[x]), cols)
        phi1[i, j] = k
        phi2[k, i] = dest_row
        phi3[dest_row, k] = dest_col
    return phi1, phi2, phi3


def bank_schedule(phi_line: np.ndarray, w: int):
    """(sigma, t) for one line of a row-wise permutation (L531-L533).

    Slot k*w + x (warp-round k, lane x) reads source s = r_k(x) = w*sigma + x
    and writes t = phi(s).
    """
    L = phi_line.size
    if L % w:
        raise ValueError("line length must be a multiple of w")
    edges = [(j % w, int(phi_line[j]) % w) for j in range(L)]
    colour = edge_colour(w, w, edges, L // w)
    sigma = np.full(L, -1, dtype=np.int64)
    t = np.full(L, -1, dtype=np.int64)
    for j in range(L):
        k = colour[j]
        x = j % w                       # source bank = lane
        slot = k * w + x
        sigma[slot] = j // w
        t[slot] = int(phi_line[j])
    return sigma, t


def make_plan(p, w: int = 32, rows: int | None = None, cols: int | None = None) -> Plan:
    p = np.asarray(p, dtype=np.int64)
    n = p.size
    if rows is None or cols is None:
        rows, cols = default_view(n)
    if rows * cols != n:
        raise ValueError("rows*cols must equal n")
    kappa = row_colouring(p, rows, cols)
    phis = phase_permutations(p, kappa, rows, cols)
    plan = Plan(n=n, rows=rows, cols=cols, w=w, kappa=kappa, phi=list(phis))
    for phi in phis:
        sig = np.empty_like(phi)
        tt = np.empty_like(phi)
        for line in range(phi.shape[0]):
            sig[line], tt[line] = bank_schedule(phi[line], w)
        plan.sigma.append(sig)
        plan.t.append(tt)
    return plan
