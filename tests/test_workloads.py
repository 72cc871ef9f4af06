"""Pins for the seeded input generators (§IV L373-L389 families).

Each family is tied to its closed form / group-theoretic identity, not to a
re-typed copy of its own formula.
"""
import numpy as np
import pytest

import workloads as W


def test_splitmix64_reference_vector():
    # Vigna's splitmix64 seeded with 0: the first output is 0xE220A8397B1DCDAF
    # (public reference value), the second 0x6E789E6AA1B965F4.
    z = W.splitmix64(0, 2)
    assert int(z[0]) == 0xE220A8397B1DCDAF
    assert int(z[1]) == 0x6E789E6AA1B965F4


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", list(range(2, 17)))
def test_families_are_permutations(fam, k):
    n = 1 << k
    p = W.make_perm(fam, n)
    assert p.dtype == np.int32 and p.size == n
    assert np.array_equal(np.sort(p), np.arange(n))


@pytest.mark.parametrize("k", [2, 5, 10, 16, 20])
def test_bitrev_is_involution(k):
    p = W.bitrev(1 << k).astype(np.int64)
    assert np.array_equal(p[p], np.arange(1 << k))


@pytest.mark.parametrize("k", [4, 8, 12, 16])
def test_bitrev_block_identity(k):
    # rev_m(i*2^{m/2} + j) = rev_{m/2}(j)*2^{m/2} + rev_{m/2}(i) for even m
    h = k // 2
    full = W.bitrev(1 << k).astype(np.int64)
    half = W.bitrev(1 << h).astype(np.int64)
    i, j = np.divmod(np.arange(1 << k), 1 << h)
    assert np.array_equal(full, half[j] * (1 << h) + half[i])


@pytest.mark.parametrize("k", [1, 2, 3, 7, 12, 15])
def test_shuffle_has_order_m(k):
    n = 1 << k
    p = W.shuffle(n).astype(np.int64)
    x = np.arange(n)
    for step in range(1, k + 1):
        x = p[x]
        if step < k:
            assert not np.array_equal(x, np.arange(n))   # order exactly m
    assert np.array_equal(x, np.arange(n))
    if k > 1:
        # perfect shuffle: index 1 -> 2, index n/2 (top bit) -> 1
        assert p[1] == 2 and p[n // 2] == 1


def test_shuffle_small_closed_form():
    # m = 3: i = (i2 i1 i0) -> (i1 i0 i2)
    assert W.shuffle(8).tolist() == [0, 2, 4, 6, 1, 3, 5, 7]


@pytest.mark.parametrize("k", [2, 4, 10, 16])
def test_square_transpose_is_involution(k):
    p = W.transpose(1 << k).astype(np.int64)
    assert np.array_equal(p[p], np.arange(1 << k))


@pytest.mark.parametrize("k", [3, 5, 11, 13])
def test_rect_transpose_matches_matrix_transpose(k):
    n = 1 << k
    R, C = W.view_shape(n)
    assert R * C == n and C == 2 * R
    p = W.transpose(n)
    a = np.arange(n)
    b = np.empty(n, dtype=np.int64)
    b[p] = a
    assert np.array_equal(b.reshape(C, R), a.reshape(R, C).T)


def test_transpose_small_closed_form():
    assert W.transpose(4).tolist() == [0, 2, 1, 3]


def test_random_is_seeded_and_distinct():
    a = W.random(4096, 42)
    b = W.random(4096, 42)
    c = W.random(4096, 43)
    assert np.array_equal(a, b)
    assert not np.array_equal(a, c)
    assert W.perm_sha256(a) == W.perm_sha256(b)


def test_random_is_uniform_on_tiny_n():
    # n = 3: each of the 3! permutations about 1/6 of the time over many seeds
    counts = {}
    for s in range(3000):
        key = tuple(W.random(4, s).tolist())
        counts[key] = counts.get(key, 0) + 1
    assert len(counts) == 24
    expect = 3000 / 24
    assert max(counts.values()) < expect * 1.6 and min(counts.values()) > expect * 0.5


def test_data_covers_special_bit_patterns():
    a = W.make_data(1 << 20)
    assert a.dtype == np.uint32
    f = a.view(np.float32)
    assert np.isnan(f).any()          # NaN payloads
    exp = (a >> 23) & 0xFF
    assert (exp == 0).any()           # subnormals / zero exponent
    a64 = W.make_data(1 << 10, 8)
    assert a64.dtype == np.uint64
    assert np.array_equal((a64 >> np.uint64(32)).astype(np.uint32), W.make_data(1 << 10, 4))
