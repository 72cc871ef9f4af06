"""The offline permutation by its definition. ORACLE — test infrastructure only.

PAPER.md L361 (§IV): "Offline permutation along P is a task to copy a[i] to
b[P(i)] for all i", with P stored in an array p, p[i] = P(i).
L365: D-designated algorithm  b[p[i]] <- a[i].
L373: S-designated algorithm  b[i] <- a[q[i]] with q = P^{-1}.

Values are moved as raw words (uint32 / uint64 views): the result is unique
and every correct implementation is bit-identical to it.
"""
from __future__ import annotations

import numpy as np


def is_perm(p: np.ndarray, n: int | None = None) -> bool:
    """P is a permutation of 0..n-1 (L361: "p[0..n-1] take distinct integers in [0, n)")."""
    p = np.asarray(p)
    if n is None:
        n = p.size
    if p.size != n:
        return False
    if n == 0:
        return True
    if p.min() < 0 or p.max() >= n:
        return False
    seen = np.zeros(n, dtype=bool)
    seen[p] = True
    return bool(seen.all())


def _words(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a)
    if a.dtype.itemsize == 4:
        return a.view(np.uint32)
    if a.dtype.itemsize == 8:
        return a.view(np.uint64)
    raise ValueError("elements must be 4 or 8 bytes")


def apply_ref(p: np.ndarray, a: np.ndarray) -> np.ndarray:
    """b with b[p[i]] = a[i] for every i (L361, L365). Raw-word copy."""
    src = _words(a)
    b = np.empty_like(src)
    b[np.asarray(p, dtype=np.int64)] = src
    return b


def inverse(p: np.ndarray) -> np.ndarray:
    """q = P^{-1}: q[p[i]] = i (L367-L373)."""
    q = np.empty_like(np.asarray(p))
    q[np.asarray(p, dtype=np.int64)] = np.arange(p.size, dtype=q.dtype)
    return q


def apply_s_designated(q: np.ndarray, a: np.ndarray) -> np.ndarray:
    """b[i] = a[q[i]] (L373). Equals apply_ref(p, a) when q = P^{-1}."""
    src = _words(a)
    return src[np.asarray(q, dtype=np.int64)].copy()


def apply_loop(p, a) -> list:
    """Pure-Python loop of the D-designated algorithm, for tiny n only (L365)."""
    b = [None] * len(a)
    for i in range(len(a)):
        b[p[i]] = a[i]
    return b
