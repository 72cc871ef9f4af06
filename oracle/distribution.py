"""Distribution D_w(P) of a permutation. ORACLE — test infrastructure only.

PAPER.md L389-L399 (§IV, formula garbled; reading F5 in DESIGN.md): the
distribution is "the total number of address groups of b accessed by all
warps in D-designated permutation algorithm":

    D_w(P) = sum_{j=0}^{n/w-1} | { floor(P(i)/w) : j*w <= i < (j+1)*w } |

so n/w <= D_w(P) <= n. L401: D_w(identical) = n/w, D_w(shuffle) = 2n/w,
D_w(bit-reversal) = D_w(transpose) = n (and the same for the inverses).
Table III (L697): 0.99987 <= D_w(P)/n <= 0.99990 for 1000 random P, n=4M.
"""
from __future__ import annotations

import numpy as np


def distribution(p: np.ndarray, w: int = 32) -> int:
    """D_w(P) exactly as defined above (warps = consecutive groups of w sources)."""
    p = np.asarray(p, dtype=np.int64)
    n = p.size
    if n % w:
        raise ValueError("n must be a multiple of w")
    g = np.sort((p // w).reshape(n // w, w), axis=1)
    distinct = 1 + (g[:, 1:] != g[:, :-1]).sum(axis=1)
    return int(distinct.sum())


def distribution_loop(p, w: int) -> int:
    """Same definition as a plain loop, for tiny n."""
    total = 0
    for j in range(len(p) // w):
        total += len({p[i] // w for i in range(j * w, (j + 1) * w)})
    return total


def expected_random_ratio(n: int, w: int = 32) -> float:
    """E[D_w(P)]/n for P uniform over all n! permutations (a closed form, not
    from the paper): each of the n/w destination groups of b is hit by a warp
    with probability 1 - C(n-w, w)/C(n, w); summing over the n/w warps gives
    E[D_w] = (n/w)^2 * (1 - prod_{k<w} (n-w-k)/(n-k))."""
    miss = 1.0
    for k in range(w):
        miss *= (n - w - k) / (n - k)
    return (n / w) * (n / w) * (1.0 - miss) / n
