"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no colouring, no phases,
no schedule). It only produces the inputs the paper's experiments use:

* the five permutation families of PAPER.md §IV (L373-L389):
  identical, shuffle, random, bit-reversal, transpose;
* a data array ``a`` of raw 32-bit (or 64-bit) words.

Both ``oracle/`` and the product tests / bench import it; neither side
imports the other.

Readings of garbled passages:
* shuffle (L373, formula garbled): rotate the m-bit index left by one bit,
  P(i) = ((i << 1) | (i >> (m-1))) & (n-1)  (perfect shuffle).
* bit-reversal (L375-L389): reverse all m bits of i.
* transpose (L389): on the R x C view with R = 2^floor(m/2), C = 2^ceil(m/2),
  P(i*C + j) = j*R + i.
* random (L375, "selected uniformly at random"): p = stable argsort of n
  splitmix64 keys drawn from a stream seeded with ``seed``. Sorting i.i.d.
  keys yields every permutation with equal probability (ties are broken by
  index; with 64-bit keys they are negligible).
"""
from __future__ import annotations

import hashlib

import numpy as np

FAMILIES = ("identity", "shuffle", "random", "bitrev", "transpose")

_GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

DATA_SEED = 0xA5A50000


def splitmix64(seed: int, count: int, start: int = 0) -> np.ndarray:
    """Outputs ``start .. start+count-1`` of the splitmix64 stream seeded with ``seed``.

    Output k is mix(seed + (k+1)*GAMMA) with the standard splitmix64 finaliser.
    """
    k = np.arange(start + 1, start + count + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + k * _GAMMA
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def log2_exact(n: int) -> int:
    m = int(n).bit_length() - 1
    if n <= 0 or (1 << m) != n:
        raise ValueError(f"n={n} is not a power of two")
    return m


def view_shape(n: int) -> tuple[int, int]:
    """R x C view of a 1-D array of n = 2^m elements: R = 2^floor(m/2), C = 2^ceil(m/2)."""
    m = log2_exact(n)
    return 1 << (m // 2), 1 << (m - m // 2)


def identity(n: int) -> np.ndarray:
    return np.arange(n, dtype=np.int32)


def shuffle(n: int) -> np.ndarray:
    m = log2_exact(n)
    i = np.arange(n, dtype=np.int64)
    if m == 0:
        return i.astype(np.int32)
    return (((i << 1) | (i >> (m - 1))) & (n - 1)).astype(np.int32)


_REV8 = np.array([int(f"{v:08b}"[::-1], 2) for v in range(256)], dtype=np.uint32)


def bitrev(n: int) -> np.ndarray:
    """Reverse all m bits of i: the 32-bit reversal of i (bytes reversed, each byte
    through a 256-entry table), shifted right by 32 - m."""
    m = log2_exact(n)
    if m == 0:
        return np.zeros(1, dtype=np.int32)
    i = np.arange(n, dtype=np.uint32)
    out = _REV8[i & 0xFF] << 24
    out |= _REV8[(i >> 8) & 0xFF] << 16
    out |= _REV8[(i >> 16) & 0xFF] << 8
    out |= _REV8[i >> 24]
    return (out >> np.uint32(32 - m)).astype(np.int32)


def transpose(n: int) -> np.ndarray:
    rows, cols = view_shape(n)
    x = np.arange(n, dtype=np.int64)
    i, j = x // cols, x % cols
    return (j * rows + i).astype(np.int32)


def random(n: int, seed: int = 42) -> np.ndarray:
    keys = splitmix64(seed, n)
    return np.argsort(keys, kind="stable").astype(np.int32)


def make_perm(family: str, n: int, seed: int = 42) -> np.ndarray:
    """int32 array p with the offline permutation b[p[i]] = a[i]."""
    if family == "identity":
        return identity(n)
    if family == "shuffle":
        return shuffle(n)
    if family == "random":
        return random(n, seed)
    if family == "bitrev":
        return bitrev(n)
    if family == "transpose":
        return transpose(n)
    raise ValueError(f"unknown family {family!r}; expected one of {FAMILIES}")


def make_data(n: int, elem_bytes: int = 4, seed: int = DATA_SEED) -> np.ndarray:
    """Raw words: hi32 of splitmix64 output i (u32), or the full 64 bits (u64).

    Reinterpreted as float these cover NaN payloads, +-0, subnormals and Inf,
    so any value-based (not bit-based) copy shows up as a mismatch.
    """
    z = splitmix64(seed, n)
    if elem_bytes == 4:
        return (z >> np.uint64(32)).astype(np.uint32)
    if elem_bytes == 8:
        return z
    raise ValueError("elem_bytes must be 4 or 8")


def perm_sha256(p: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(p, dtype=np.int32).tobytes()).hexdigest()
