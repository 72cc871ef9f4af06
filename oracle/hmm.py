"""Memory-machine access classes. ORACLE — test infrastructure only.

PAPER.md §II-§III:
* L201 (DMM): cell m[i] lies in bank i mod w; one time unit serves cells of
  distinct banks; same-bank cells take one pipeline stage each.
* L207 (UMM): address group A[j] = {m[j*w], ..., m[(j+1)*w - 1]}; cells of
  one group are served together, each further group costs one stage.
* L213 (§III): a warp's round is *coalesced* if all addresses lie in one
  address group, *conflict-free* if any two addresses are equal or lie in
  distinct banks. "Clearly, the memory access is conflict-free if it is
  coalesced." A round that is neither is *casual*.
* Fig. 3 (L217-L357): w = 4, W0 -> {7,5,15,0}, W1 -> {10,11,12,9}: the DMM
  needs 3 stages, the UMM 5.
"""
from __future__ import annotations

import numpy as np


def dmm_stages(warp_addrs, w: int) -> int:
    """Pipeline stages one warp occupies on the DMM: the largest number of
    DISTINCT addresses that fall in one bank (L201, Fig. 3)."""
    addrs = set(int(x) for x in warp_addrs)
    per_bank: dict[int, int] = {}
    for x in addrs:
        per_bank[x % w] = per_bank.get(x % w, 0) + 1
    return max(per_bank.values()) if per_bank else 0


def umm_stages(warp_addrs, w: int) -> int:
    """Pipeline stages one warp occupies on the UMM: the number of distinct
    address groups it touches (L207, Fig. 3)."""
    return len({int(x) // w for x in warp_addrs})


def is_coalesced(warp_addrs, w: int) -> bool:
    """L213: floor(a_0/w) = floor(a_1/w) = ... = floor(a_{w-1}/w)."""
    return umm_stages(warp_addrs, w) <= 1


def is_conflict_free(warp_addrs, w: int) -> bool:
    """L213: for all i<j, a_i = a_j or a_i mod w != a_j mod w."""
    return dmm_stages(warp_addrs, w) <= 1


def classify_round(addrs: np.ndarray, w: int) -> str:
    """Classify a whole round (every thread one access, threads grouped into
    consecutive warps of w) as 'coalesced', 'conflict-free' or 'casual'
    (L213-L215). A round is coalesced/conflict-free iff every warp is."""
    a = np.asarray(addrs, dtype=np.int64).reshape(-1, w)
    groups = a // w
    if np.all(groups == groups[:, :1]):
        return "coalesced"
    banks = a % w
    # conflict-free: equal banks only for equal addresses
    ok = True
    for row_a, row_b in zip(a, banks):
        if dmm_stages(row_a, w) > 1:
            ok = False
            break
    return "conflict-free" if ok else "casual"


def classify_round_fast(addrs: np.ndarray, w: int) -> str:
    """Vectorised classify_round for large rounds (same definition)."""
    a = np.asarray(addrs, dtype=np.int64).reshape(-1, w)
    groups = a // w
    if np.all(groups == groups[:, :1]):
        return "coalesced"
    s = np.sort(a, axis=1)
    # distinct addresses per warp, then check their banks are distinct
    keep = np.ones_like(s, dtype=bool)
    keep[:, 1:] = s[:, 1:] != s[:, :-1]
    banks = np.where(keep, s % w, -1 - np.arange(w)[None, :])  # drop duplicates
    bs = np.sort(banks, axis=1)
    dup = (bs[:, 1:] == bs[:, :-1]) & (bs[:, 1:] >= 0)
    return "casual" if dup.any() else "conflict-free"
