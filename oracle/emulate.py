"""Paper-faithful emulation of the algorithms on the HMM. ORACLE — test infrastructure only.

Executes, on numpy arrays, exactly the steps PAPER.md spells out, and records
every round of memory access with its class (L211-L215) so that Table I can
be reproduced by counting:

* transpose (§V, Lemma 5): diagonal arrangement
  c[i][(i+j) mod w] <- a[i][j]; b[i][j] <- c[j][(i+j) mod w], per w x w block
  A_{I,J} -> B_{J,I};
* row-wise permutation (§VI, Lemma 7): Step 1 A_i[j] <- a[i][j];
  Step 2 s <- s[i][j], t <- t[i][j]; Step 3 B_i[t] <- A_i[s];
  Step 4 b[i][j] <- B_i[j];
* column-wise permutation (Lemma 8): transpose, row-wise, transpose;
* scheduled permutation (§VII, Thm 9): row-wise, column-wise, row-wise
  = R, T, R, T, R (the paper's "five sequential kernel calls", L699);
* D-designated (L365) and S-designated (L373) algorithms.

Table I (L377-L407): scheduled = 11 coalesced global reads, 5 coalesced
global writes, 8 conflict-free shared reads, 8 conflict-free shared writes.
"""
from __future__ import annotations

from collections import Counter

import numpy as np

from .hmm import classify_round_fast


class Rounds:
    """Counter of memory-access rounds keyed by (memory, op, class)."""

    def __init__(self, w: int):
        self.w = w
        self.c = Counter()

    def glob(self, op: str, addrs: np.ndarray):
        cls = classify_round_fast(np.asarray(addrs).ravel(), self.w)
        self.c[("global", op, "coalesced" if cls == "coalesced" else "casual")] += 1

    def shared(self, op: str, addrs: np.ndarray):
        # shared addresses are per-block indices; warps = w consecutive threads
        cls = classify_round_fast(np.asarray(addrs).ravel(), self.w)
        self.c[("shared", op, "conflict-free" if cls != "casual" else "conflicting")] += 1

    def table(self) -> dict:
        return dict(self.c)


def row_wise(X: np.ndarray, sigma: np.ndarray, t: np.ndarray, w: int, rc: Rounds) -> np.ndarray:
    """Row-wise permutation of X (lines x L) with schedule s = w*sigma + lane, t (L521-L525)."""
    lines, L = X.shape
    j = np.arange(L, dtype=np.int64)[None, :].repeat(lines, 0)
    i = np.arange(lines, dtype=np.int64)[:, None].repeat(L, 1)
    # Step 1: A_i[j] <- a[i][j]
    rc.glob("read", i * L + j)
    A = X.copy()
    rc.shared("write", j)
    # Step 2: s <- s[i][j], t <- t[i][j]   (two global arrays, coalesced)
    rc.glob("read", i * L + j)
    rc.glob("read", i * L + j)
    s = w * np.asarray(sigma, dtype=np.int64) + (j % w)
    tt = np.asarray(t, dtype=np.int64)
    # Step 3: B_i[t] <- A_i[s]
    rc.shared("read", s)
    B = np.empty_like(A)
    vals = np.take_along_axis(A, s, axis=1)
    rc.shared("write", tt)
    np.put_along_axis(B, tt, vals, axis=1)
    # Step 4: b[i][j] <- B_i[j]
    rc.shared("read", j)
    rc.glob("write", i * L + j)
    return B


def diagonal_address(i, j, w: int):
    """Diagonal arrangement (L409-L415, Fig. 4): element (i, j) of a w x w tile
    is stored at shared address i*w + (i+j) mod w, so every row and every
    column of the tile occupies w distinct banks."""
    return i * w + (i + j) % w


def transpose(X: np.ndarray, w: int, rc: Rounds) -> np.ndarray:
    """Blocked transpose with the diagonal arrangement (L409-L423)."""
    R, C = X.shape
    if R % w or C % w:
        raise ValueError("matrix sides must be multiples of w")
    I, J, ii, jj = np.meshgrid(np.arange(R // w), np.arange(C // w), np.arange(w),
                               np.arange(w), indexing="ij")
    # thread (i, j) of the block for A_{I,J}; a warp = fixed (I, J, i), lanes j
    # Step 1: c[i][(i+j) mod w] <- a[I*w+i][J*w+j]
    rc.glob("read", (I * w + ii) * C + J * w + jj)
    rc.shared("write", diagonal_address(ii, jj, w))
    tile = X.reshape(R // w, w, C // w, w).transpose(0, 2, 1, 3)      # [I][J][i][j]
    cbuf = np.empty_like(tile)
    np.put_along_axis(cbuf, (ii + jj) % w, tile, axis=3)              # c[i][(i+j)%w]
    # Step 2: b[J*w+i][I*w+j] <- c[j][(i+j) mod w]
    rc.shared("read", diagonal_address(jj, ii, w))
    vals = cbuf[I, J, jj, (ii + jj) % w]
    rc.glob("write", (J * w + ii) * R + I * w + jj)
    Y = np.empty((C, R), dtype=X.dtype)
    Y[J * w + ii, I * w + jj] = vals
    return Y


def scheduled(a: np.ndarray, sched, rows: int, cols: int, w: int, rc: Rounds | None = None):
    """Row-wise, column-wise (= T, R, T), row-wise (Thm 9; L699)."""
    rc = rc or Rounds(w)
    X = np.asarray(a).reshape(rows, cols)
    (s1, t1), (s2, t2), (s3, t3) = sched
    X = row_wise(X, s1, t1, w, rc)          # step 1
    X = transpose(X, w, rc)                 # step 2 = T, R, T
    X = row_wise(X, s2, t2, w, rc)
    X = transpose(X, w, rc)
    X = row_wise(X, s3, t3, w, rc)          # step 3
    return X.reshape(-1), rc


def d_designated(p: np.ndarray, a: np.ndarray, w: int, rc: Rounds | None = None):
    """b[p[i]] <- a[i] for all i (L365, Lemma 2)."""
    rc = rc or Rounds(w)
    n = a.size
    idx = np.arange(n, dtype=np.int64)
    rc.glob("read", idx)            # a[i]
    rc.glob("read", idx)            # p[i]
    rc.glob("write", np.asarray(p, dtype=np.int64))
    b = np.empty_like(a)
    b[np.asarray(p, dtype=np.int64)] = a
    return b, rc


def s_designated(q: np.ndarray, a: np.ndarray, w: int, rc: Rounds | None = None):
    """b[i] <- a[q[i]] for all i (L373, Lemma 3)."""
    rc = rc or Rounds(w)
    n = a.size
    idx = np.arange(n, dtype=np.int64)
    rc.glob("read", idx)            # q[i]
    rc.glob("read", np.asarray(q, dtype=np.int64))
    rc.glob("write", idx)
    return a[np.asarray(q, dtype=np.int64)].copy(), rc
