"""Pins for the reference planner, checker and paper-faithful emulator.

* Fig. 6 (L539-L679): the paper's own colouring passes the checker, and the
  emulator reproduces its three intermediate matrices.
* Fig. 4 (L427-L495): the diagonal-arrangement address map.
* Table I (L377-L407): round counts of every algorithm, scheduled = 11/5/8/8.
* Thm 6 (L515) by brute force: every permutation of n = 4 and n = 8 (2x4,
  4x2, w = 2) decomposes, and the emulator then computes b[P(i)] = a[i].
* The checker itself is pinned by mutation: corrupting a valid plan in each
  way the invariants name makes the corresponding invariant fail.
"""
import itertools
import json
import os

import numpy as np
import pytest

import workloads as W
from oracle import apply as OA
from oracle import check as OC
from oracle import emulate as OE
from oracle import konig as OK
from oracle import planner as OP

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def sched_of(plan):
    return list(zip(plan.sigma, plan.t))


# ---------------------------------------------------------------- König (Thm 6)

def test_konig_colours_regular_multigraphs():
    rng = np.random.default_rng(0)
    for deg in (1, 2, 3, 4, 8):
        for nodes in (2, 3, 5, 8):
            # random d-regular bipartite multigraph = union of d random perfect matchings
            edges = []
            for _ in range(deg):
                perm = rng.permutation(nodes)
                edges += [(u, int(perm[u])) for u in range(nodes)]
            order = rng.permutation(len(edges))
            edges = [edges[i] for i in order]
            col = OK.edge_colour(nodes, nodes, edges, deg)
            assert OK.is_proper(nodes, nodes, edges, col, deg)


def test_konig_fig5_shape():
    # Fig. 5 (L527-L529): a 4-regular bipartite graph painted with 4 colours
    edges = [(u, (u + s) % 4) for u in range(4) for s in range(4)]
    col = OK.edge_colour(4, 4, edges, 4)
    assert OK.is_proper(4, 4, edges, col, 4)
    assert sorted(col) == sorted([c for c in range(4) for _ in range(4)])


# ---------------------------------------------------------------- Fig. 4

def test_fig4_diagonal_arrangement():
    g = gold("fig4.json")
    w = g["w"]
    holds = [None] * (w * w)
    for i in range(w):
        for j in range(w):
            holds[OE.diagonal_address(i, j, w)] = [i, j]
    assert holds == g["address_holds"]
    # every row and every column of the tile occupies w distinct banks (L415)
    for i in range(w):
        assert len({OE.diagonal_address(i, j, w) % w for j in range(w)}) == w
        assert len({OE.diagonal_address(j, i, w) % w for j in range(w)}) == w


# ---------------------------------------------------------------- Fig. 6

def _fig6():
    g = gold("fig6.json")
    s = g["sqrt_n"]
    lab = np.array(g["input"])                # [row][col] -> (dest row, dest col)
    p = (lab[..., 0] * s + lab[..., 1]).reshape(-1)
    return g, s, p


def test_fig6_paper_colouring_passes_checker():
    g, s, p = _fig6()
    after1 = np.array(g["after_step1"])
    lab = np.array(g["input"])
    # the paper's colouring: an element's colour is its column after Step 1 (L537-L539)
    kappa = np.empty(s * s, dtype=np.int64)
    for i in range(s):
        for j in range(s):
            k = [c for c in range(s) if tuple(after1[i, c]) == tuple(lab[i, j])]
            assert len(k) == 1
            kappa[i * s + j] = k[0]
    assert kappa.reshape(s, s).tolist() == [[1, 2, 0, 3], [0, 1, 3, 2], [2, 0, 1, 3], [3, 0, 1, 2]]
    phis = OC.phases_from_kappa(p, kappa, s, s)
    w = 2
    sched = []
    for ph in phis:
        sig = np.empty_like(ph)
        tt = np.empty_like(ph)
        for line in range(ph.shape[0]):
            sig[line], tt[line] = OP.bank_schedule(ph[line], w)
        sched.append((sig, tt))
    OC.assert_plan(p, kappa, sched, s, s, w)
    # the emulator driven by this plan reproduces the paper's intermediate matrices
    rc = OE.Rounds(w)
    a = np.arange(s * s, dtype=np.int64)            # a[x] = x, so values are element ids
    label = lab.reshape(-1, 2)
    X = OE.row_wise(a.reshape(s, s), *sched[0], w, rc)
    assert (label[X]).tolist() == g["after_step1"]
    X = OE.transpose(X, w, rc)
    X = OE.row_wise(X, *sched[1], w, rc)
    X = OE.transpose(X, w, rc)
    assert (label[X]).tolist() == g["after_step2"]
    X = OE.row_wise(X, *sched[2], w, rc)
    assert (label[X]).tolist() == g["after_step3"]


def test_fig6_reference_planner():
    g, s, p = _fig6()
    plan = OP.make_plan(p, w=2)
    OC.assert_plan(p, plan.kappa, sched_of(plan), s, s, 2)
    a = W.make_data(16)
    b, _ = OE.scheduled(a, sched_of(plan), s, s, 2)
    assert np.array_equal(b, OA.apply_ref(p, a))


# ---------------------------------------------------------------- Table I

def _tbl(rc):
    t = rc.table()
    return [t.get(("global", "read", "casual"), 0), t.get(("global", "write", "casual"), 0),
            t.get(("global", "read", "coalesced"), 0), t.get(("global", "write", "coalesced"), 0),
            t.get(("shared", "read", "conflict-free"), 0),
            t.get(("shared", "write", "conflict-free"), 0)]


@pytest.mark.parametrize("fam", W.FAMILIES)
def test_table1_round_counts(fam):
    g = gold("table1.json")["rows"]
    n, w = 1 << 12, 32
    p = W.make_perm(fam, n)
    a = W.make_data(n)
    plan = OP.make_plan(p, w=w)
    OC.assert_plan(p, plan.kappa, sched_of(plan), plan.rows, plan.cols, w)
    b, rc = OE.scheduled(a, sched_of(plan), plan.rows, plan.cols, w)
    assert np.array_equal(b, OA.apply_ref(p, a))
    assert _tbl(rc) == g["scheduled"]
    assert sum(_tbl(rc)) == gold("table1.json")["scheduled_total_rounds"]
    assert rc.table().get(("shared", "read", "conflicting"), 0) == 0
    assert rc.table().get(("shared", "write", "conflicting"), 0) == 0
    # the pieces (Lemmas 5, 7, 8)
    X = a.reshape(plan.rows, plan.cols)
    rcT = OE.Rounds(w)
    OE.transpose(X, w, rcT)
    assert _tbl(rcT) == g["transpose"]
    rcR = OE.Rounds(w)
    OE.row_wise(X, plan.sigma[0], plan.t[0], w, rcR)
    assert _tbl(rcR) == g["row_wise"]
    rcC = OE.Rounds(w)
    Y = OE.transpose(X, w, rcC)
    Y = OE.row_wise(Y, plan.sigma[1], plan.t[1], w, rcC)
    OE.transpose(Y, w, rcC)
    assert _tbl(rcC) == g["column_wise"]


def test_table1_conventional_round_counts():
    g = gold("table1.json")["rows"]
    n, w = 1 << 12, 32
    a = W.make_data(n)
    for fam in ("random", "bitrev", "transpose"):     # large distribution: casual access
        p = W.make_perm(fam, n)
        b, rc = OE.d_designated(p, a, w)
        assert np.array_equal(b, OA.apply_ref(p, a)) and _tbl(rc) == g["d_designated"]
        b, rc = OE.s_designated(OA.inverse(p), a, w)
        assert np.array_equal(b, OA.apply_ref(p, a)) and _tbl(rc) == g["s_designated"]
    # identical: every access happens to be coalesced (Lemma 4, D_w = n/w)
    _, rc = OE.d_designated(W.identity(n), a, w)
    assert rc.table()[("global", "write", "coalesced")] == 1


# ---------------------------------------------------------------- brute force (Thm 6)

@pytest.mark.parametrize("rows,cols", [(2, 2), (2, 4), (4, 2)])
def test_bruteforce_all_permutations_decompose(rows, cols):
    n, w = rows * cols, 2
    a = np.arange(100, 100 + n, dtype=np.uint32)
    count = 0
    for perm in itertools.permutations(range(n)):
        p = np.array(perm, dtype=np.int64)
        plan = OP.make_plan(p, w=w, rows=rows, cols=cols)
        sched = sched_of(plan)
        res = OC.check_plan(p, plan.kappa, sched, rows, cols, w)
        assert all(res.values()), (perm, res)
        if count % 17 == 0:      # the full emulator on a deterministic subsample
            b, _ = OE.scheduled(a, sched, rows, cols, w)
            assert np.array_equal(b, OA.apply_ref(p, a)), perm
        count += 1
    assert count == int(np.prod(range(1, n + 1)))


def test_sampled_3x3_decomposes():
    # n = 9, 3 x 3 view, w = 3 (not a power of two: exercises the general König)
    rng = np.random.default_rng(9)
    a = np.arange(9, dtype=np.uint32)
    for _ in range(300):
        p = rng.permutation(9)
        plan = OP.make_plan(p, w=3, rows=3, cols=3)
        OC.assert_plan(p, plan.kappa, sched_of(plan), 3, 3, 3)
        b, rc = OE.scheduled(a, sched_of(plan), 3, 3, 3)
        assert np.array_equal(b, OA.apply_ref(p, a))


@pytest.mark.parametrize("k", [10, 11, 13])
def test_reference_planner_families(k):
    n, w = 1 << k, 32
    rows, cols = W.view_shape(n)
    if rows < w:
        pytest.skip("view narrower than w")
    a = W.make_data(n)
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n)
        plan = OP.make_plan(p, w=w)
        OC.assert_plan(p, plan.kappa, sched_of(plan), rows, cols, w)
        b, _ = OE.scheduled(a, sched_of(plan), rows, cols, w)
        assert np.array_equal(b, OA.apply_ref(p, a))


# ---------------------------------------------------------------- checker mutations

def test_checker_rejects_each_kind_of_corruption():
    n, w = 1 << 12, 32
    p = W.random(n, 11)
    plan = OP.make_plan(p, w=w)
    r, c = plan.rows, plan.cols
    good = sched_of(plan)
    assert all(OC.check_plan(p, plan.kappa, good, r, c, w).values())

    # (i)/(ii): swap the colours of two elements in different rows
    k2 = plan.kappa.copy()
    k2[0], k2[c] = k2[c], k2[0]
    res = OC.check_plan(p, k2, good, r, c, w)
    if k2[0] != k2[c]:
        assert not (res["i_row_colours_bijective"] and res["ii_colour_dest_rows_distinct"])
    # (i): duplicate a colour inside one row
    k3 = plan.kappa.copy()
    k3[1] = k3[0]
    assert not OC.check_plan(p, k3, good, r, c, w)["i_row_colours_bijective"]

    # (v): wrong destination in one slot
    s1, t1 = good[0][0].copy(), good[0][1].copy()
    t1[0, 0] = (t1[0, 0] + 1) % c
    res = OC.check_plan(p, plan.kappa, [(s1, t1), good[1], good[2]], r, c, w)
    assert not res["v_t_equals_phi_of_s"]

    # (vii): point one slot at a source that another slot already reads
    s2, t2 = good[1][0].copy(), good[1][1].copy()
    s2[0, 0] = (s2[0, 0] + 1) % (r // w)
    res = OC.check_plan(p, plan.kappa, [good[0], (s2, t2), good[2]], r, c, w)
    assert not res["vii_sources_cover_line"] and not res["v_t_equals_phi_of_s"]

    # (vi) specifically: exchange t between two lanes of different rounds keeping (v)
    s3, t3 = good[2][0].copy(), good[2][1].copy()
    # slots (round 0, lane x) and (round 1, lane x) both read bank x: swapping the
    # pair keeps every t = Phi(s) and the coverage, only the round membership changes
    x = 0
    a0, a1 = x, w + x
    s3[0, a0], s3[0, a1] = s3[0, a1], s3[0, a0]
    t3[0, a0], t3[0, a1] = t3[0, a1], t3[0, a0]
    res = OC.check_plan(p, plan.kappa, [good[0], good[1], (s3, t3)], r, c, w)
    assert res["v_t_equals_phi_of_s"] and res["vii_sources_cover_line"]
    if (t3[0, a0] % w) != (t3[0, a1] % w):
        assert not res["vi_rounds_conflict_free"]

    # (iv): a plan for a different permutation
    p2 = p.copy()
    p2[0], p2[1] = p2[1], p2[0]
    res = OC.check_plan(p2, plan.kappa, good, r, c, w)
    assert not all(res.values())
