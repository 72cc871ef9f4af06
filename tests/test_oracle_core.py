"""Pins for oracle/apply.py, oracle/hmm.py, oracle/distribution.py.

Each check ties the oracle to something other than itself: the paper's
printed values (Fig. 3, Table III), closed forms (L401), the matrix
transpose / bit-reversal identities, a pure-Python loop on tiny inputs.
"""
import json
import os

import numpy as np
import pytest

import workloads as W
from oracle import apply as OA
from oracle import distribution as OD
from oracle import hmm as OH

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- apply (L361)

def test_apply_matches_python_loop():
    for k in (1, 3, 6):
        n = 1 << k
        for fam in W.FAMILIES:
            p = W.make_perm(fam, n, seed=7)
            a = W.make_data(n)
            assert OA.apply_ref(p, a).tolist() == OA.apply_loop(p.tolist(), a.tolist())


def test_apply_identity_is_copy():
    a = W.make_data(1 << 12)
    assert np.array_equal(OA.apply_ref(W.identity(a.size), a), a)


@pytest.mark.parametrize("k", [4, 9, 12])
def test_apply_transpose_is_matrix_transpose(k):
    n = 1 << k
    R, C = W.view_shape(n)
    a = W.make_data(n)
    b = OA.apply_ref(W.transpose(n), a)
    assert np.array_equal(b.reshape(C, R), a.reshape(R, C).T)


def test_apply_bitrev_closed_form():
    n = 1 << 10
    a = W.make_data(n)
    b = OA.apply_ref(W.bitrev(n), a)
    # b[rev(i)] = a[i]  <=>  b[j] = a[rev(j)] (rev is an involution)
    rev = np.array([int(format(i, "010b")[::-1], 2) for i in range(n)])
    assert np.array_equal(b, a[rev])


def test_apply_shuffle_closed_form():
    n = 1 << 8
    a = W.make_data(n)
    b = OA.apply_ref(W.shuffle(n), a)
    # shuffle sends the lower half to even slots and the upper half to odd slots
    assert np.array_equal(b[0::2], a[: n // 2])
    assert np.array_equal(b[1::2], a[n // 2:])


def test_apply_is_bitwise_on_nan_payloads():
    a = np.array([0x7FC00001, 0xFFFFFFFF, 0x80000000, 0x00000001, 0x7F800000, 0, 1, 2],
                 dtype=np.uint32)
    p = np.array([3, 0, 7, 1, 6, 2, 5, 4], dtype=np.int32)
    b = OA.apply_ref(p, a.view(np.float32))
    assert b.dtype == np.uint32
    expect = np.empty(8, dtype=np.uint32)
    for i in range(8):
        expect[p[i]] = a[i]
    assert np.array_equal(b, expect)


def test_s_designated_equals_d_designated():
    n = 1 << 12
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n)
        a = W.make_data(n)
        q = OA.inverse(p)
        assert np.array_equal(OA.apply_s_designated(q, a), OA.apply_ref(p, a))


def test_is_perm():
    assert OA.is_perm(np.array([2, 0, 1]))
    assert not OA.is_perm(np.array([2, 0, 0]))
    assert not OA.is_perm(np.array([3, 0, 1]))
    assert not OA.is_perm(np.array([-1, 0, 1]))


def test_c_loop_matches_definition():
    from oracle import capply
    n = 1 << 14
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n)
        a = W.make_data(n)
        assert np.array_equal(capply.apply_c(p, a), OA.apply_ref(p, a))
    a8 = W.make_data(n, 8)
    p = W.random(n, 3)
    assert np.array_equal(capply.apply_c(p, a8), OA.apply_ref(p, a8))
    assert capply.threads() >= 1


# ---------------------------------------------------------------- hmm (L201-L215, Fig. 3)

def test_fig3_stage_counts():
    g = gold("fig3.json")
    w = g["w"]
    dmm = [OH.dmm_stages(wa, w) for wa in g["warps"]]
    umm = [OH.umm_stages(wa, w) for wa in g["warps"]]
    assert dmm == g["dmm_stages"] and sum(dmm) == g["dmm_total_stages"]
    assert umm == g["umm_stages"] and sum(umm) == g["umm_total_stages"]


def test_access_classes():
    w = 4
    assert OH.is_coalesced([4, 5, 6, 7], w) and OH.is_conflict_free([4, 5, 6, 7], w)
    assert OH.is_conflict_free([0, 5, 10, 15], w) and not OH.is_coalesced([0, 5, 10, 15], w)
    assert OH.is_conflict_free([3, 3, 3, 3], w)          # broadcast (a_i = a_j)
    assert not OH.is_conflict_free([3, 7, 0, 1], w)      # 3 and 7 share bank 3
    assert OH.classify_round(np.array([0, 1, 2, 3, 8, 9, 10, 11]), w) == "coalesced"
    assert OH.classify_round(np.array([0, 5, 10, 15, 1, 2, 3, 0]), w) == "conflict-free"
    assert OH.classify_round(np.array([0, 4, 1, 2, 1, 2, 3, 0]), w) == "casual"
    rng = np.random.default_rng(0)
    for _ in range(200):
        x = rng.integers(0, 64, size=32)
        assert OH.classify_round(x, 8) == OH.classify_round_fast(x, 8)


# ---------------------------------------------------------------- D_w (L389-L401, Table III)

@pytest.mark.parametrize("k", [10, 12, 16, 20])
def test_distribution_closed_forms(k):
    n, w = 1 << k, 32
    assert OD.distribution(W.identity(n), w) == n // w
    assert OD.distribution(W.shuffle(n), w) == 2 * n // w
    assert OD.distribution(OA.inverse(W.shuffle(n)), w) == 2 * n // w
    assert OD.distribution(W.bitrev(n), w) == n
    if k % 2 == 0:
        assert OD.distribution(W.transpose(n), w) == n
        assert OD.distribution(OA.inverse(W.transpose(n)), w) == n


def test_distribution_matches_loop():
    for fam in W.FAMILIES:
        p = W.make_perm(fam, 256, seed=5)
        for w in (2, 4, 8, 32):
            assert OD.distribution(p, w) == OD.distribution_loop(p.tolist(), w)


def test_distribution_bounds():
    rng = np.random.default_rng(1)
    for _ in range(20):
        p = rng.permutation(1024)
        d = OD.distribution(p, 32)
        assert 1024 // 32 <= d <= 1024


def test_expected_random_ratio_inside_table3_band():
    g = gold("table3.json")
    e = OD.expected_random_ratio(g["n"], g["w"])
    assert abs(e - 0.9998854) < 1e-7
    assert g["dw_over_n"]["min"] <= round(e, 5) <= g["dw_over_n"]["max"]


def test_table3_distribution_of_random_permutations():
    g = gold("table3.json")
    n, w = g["n"], g["w"]
    tol = g["printed_precision"] / 2
    vals = [OD.distribution(W.random(n, 42 + s), w) / n for s in range(6)]
    for v in vals:
        assert g["dw_over_n"]["min"] - tol <= v <= g["dw_over_n"]["max"] + tol
    e = OD.expected_random_ratio(n, w)
    sd = 6e-6   # ~sqrt(#collisions)/n for n = 4M, w = 32
    assert abs(np.mean(vals) - e) < 3 * sd
