"""Pins of the oracle's tiled forms (oracle/tiled.py) and of their checkers
(oracle/check.py check_tlc / check_cluster), independently of the product.

* The oracle BUILDS TLC and cluster plans itself (its own König colourings by alternating
  paths, elements followed through the passes) and EXECUTES plans with a chunk-scatter /
  block-exchange description of the storage; the executed result must equal the
  definition b[P(i)] = a[i] and every round must be conflict-free
  (L531-L533). The checkers, which derive each element from its source offset with
  their own formulas, must accept those plans -- so a wrong layout formula in a checker
  (swapped h1/h2, a transposed chunk, a wrong sender index) fails here, not only when a
  product plan disagrees.
* Mutations of a valid plan (a swapped destination, a moved lane, a round made
  conflicting) must be rejected by the checker and change the executed output.
* The product's exported TLC plans run through the ORACLE's executor and reach
  b[P(i)] = a[i].
"""
import itertools

import numpy as np
import pytest

import workloads as W
from oracle import apply as OA
from oracle import check as OC
from oracle import tiled as OT


def _ok(res):
    return all(res.values()) and len(res) >= 8


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k,h", [(10, (2, 4, 2)), (12, (2, 4, 8)), (12, (8, 4, 2)), (12, (4, 4, 4))])
def test_oracle_tlc_plan_executes_and_checks(fam, k, h):
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm(fam, n, seed=k)
    kappa, sched = OT.tlc_plan(p, r, c, h)
    a = W.make_data(n)
    b, st = OT.tlc_apply(a, sched, r, c, h)
    assert np.array_equal(b, OA.apply_ref(p, a))
    assert st["rounds"] == 3 * n // 32 == st["conflict_free"]
    assert _ok(OC.check_tlc(p, kappa, sched, r, c, h))


def test_check_tlc_rejects_wrong_layout_parameters():
    # a checker that confused h1 with h3 or h2 would reject the oracle's own plan
    n = 1 << 12
    r, c = W.view_shape(n)
    p = W.random(n, 1)
    h = (2, 4, 8)
    kappa, sched = OT.tlc_plan(p, r, c, h)
    assert _ok(OC.check_tlc(p, kappa, sched, r, c, h))
    for wrong in ((8, 4, 2), (4, 2, 8), (2, 8, 4)):
        with pytest.raises(Exception):
            assert _ok(OC.check_tlc(p, kappa, sched, r, c, wrong))


def test_check_tlc_and_executor_reject_mutations():
    n = 1 << 12
    r, c = W.view_shape(n)
    p = W.random(n, 2)
    h = (4, 4, 4)
    a = W.make_data(n)
    kappa, sched = OT.tlc_plan(p, r, c, h)
    ref = OA.apply_ref(p, a)
    # (1) two destinations of one round swapped: still a bijection, wrong mapping
    bad = [s.copy() for s in sched]
    e0, e1 = int(bad[1][0]), int(bad[1][1])
    bad[1][0] = (e0 & 0xFFFF0000) | (e1 & 0xFFFF)
    bad[1][1] = (e1 & 0xFFFF0000) | (e0 & 0xFFFF)
    res = OC.check_tlc(p, kappa, bad, r, c, h)
    assert not res["v_tiles_implement_phi"]
    assert not np.array_equal(OT.tlc_apply(a, bad, r, c, h)[0], ref)
    # (2) two whole entries with the same lane moved between rounds 0 and 1: every entry
    # still maps its own element (lane, mapping and coverage hold) but round 0 now
    # writes one bank twice
    bad = [s.copy() for s in sched]
    t0 = bad[0]
    dbank = lambda slot: int(t0[slot]) & 31
    x = next(x for x in range(32) if dbank(32 + x) != dbank(x))
    t0[x], t0[32 + x] = t0[32 + x], t0[x]
    res = OC.check_tlc(p, kappa, bad, r, c, h)
    assert res["viii_lane_is_source_bank"] and res["v_tiles_implement_phi"]
    assert not res["vi_rounds_conflict_free_A_and_B"]
    b, st = OT.tlc_apply(a, bad, r, c, h)
    assert np.array_equal(b, ref) and st["conflict_free"] == st["rounds"] - 2


def test_tlc_bruteforce_tiny_w2():
    # n = 8 as a 2 x 4 view, w = 2, tiles (1, 2, 1): a sample of all 8! permutations
    n, r, c, h, w = 8, 2, 4, (1, 2, 1), 2
    a = np.arange(100, 100 + n, dtype=np.uint32)
    for perm in itertools.islice(itertools.permutations(range(n)), 0, 40320, 37):
        p = np.array(perm, dtype=np.int64)
        kappa, sched = OT.tlc_plan(p, r, c, h, w)
        b, st = OT.tlc_apply(a, sched, r, c, h, w)
        assert np.array_equal(b, OA.apply_ref(p, a)), perm
        assert st["conflict_free"] == st["rounds"]
        assert _ok(OC.check_tlc(p, kappa, sched, r, c, h, w))


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k,C", [(10, 2), (12, 2), (12, 4), (14, 4)])
def test_oracle_cluster_plan_executes_and_checks(fam, k, C):
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm(fam, n, seed=k + C)
    kappa, sched = OT.cluster_plan(p, r, c, C)
    a = W.make_data(n)
    b, st = OT.cluster_apply(a, sched, r, c, C)
    assert np.array_equal(b, OA.apply_ref(p, a))
    assert st["rounds"] == 3 * n // 32 == st["conflict_free"]
    assert _ok(OC.check_cluster(p, kappa, sched, r, c, C))


def test_check_cluster_rejects_wrong_block_count_and_mutations():
    n = 1 << 12
    r, c = W.view_shape(n)
    p = W.random(n, 9)
    kappa, sched = OT.cluster_plan(p, r, c, 4)
    assert _ok(OC.check_cluster(p, kappa, sched, r, c, 4))
    assert not _ok(OC.check_cluster(p, kappa, sched, r, c, 2))
    bad = [s.copy() for s in sched]
    e0, e1 = int(bad[2][5]), int(bad[2][6])
    bad[2][5] = (e0 & 0xFFFF0000) | (e1 & 0xFFFF)
    bad[2][6] = (e1 & 0xFFFF0000) | (e0 & 0xFFFF)
    assert not OC.check_cluster(p, kappa, bad, r, c, 4)["v_blocks_implement_phi"]
    a = W.make_data(n)
    assert not np.array_equal(OT.cluster_apply(a, bad, r, c, 4)[0], OA.apply_ref(p, a))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_kasagini13_b200 import build
    build.build()
    import paper_conf_icpp_kasagini13_b200 as P
    return P


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [15, 16])
def test_product_tlc_plan_runs_on_the_oracle_executor(lib, fam, k):
    n = 1 << k
    p = W.make_perm(fam, n, seed=3 * k)
    with lib.Plan(p, device=False, passes=3, layout=3, direct=-1) as pl:
        info = pl.info()
        _, scheds = pl.export()
    r, c = info["rows"], info["cols"]
    h = tuple(info["h"])
    a = W.make_data(n)
    b, st = OT.tlc_apply(a, [s.reshape(-1) for s in scheds], r, c, h)
    assert np.array_equal(b, OA.apply_ref(p, a))
    assert st["conflict_free"] == st["rounds"] == 3 * n // 32


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k,C", [(15, 8), (15, 16), (16, 16), (17, 16), (18, 16), (16, 4)])
def test_product_cluster_plan_checks_and_runs_on_the_oracle_executor(lib, fam, k, C):
    n = 1 << k
    p = W.make_perm(fam, n, seed=k + C)
    with lib.Plan(p, device=False, passes=2, cluster=C, direct=-1) as pl:
        info = pl.info()
        d = pl.describe()
        kappa, scheds = pl.export()
    assert info["passes"] == 2 and d["cluster"] == C and info["kernels_per_apply"] == 1
    r, c = info["rows"], info["cols"]
    sched = [s.reshape(-1) for s in scheds]
    assert _ok(OC.check_cluster(p, kappa.astype(np.int64), sched, r, c, C))
    a = W.make_data(n)
    b, st = OT.cluster_apply(a, sched, r, c, C)
    assert np.array_equal(b, OA.apply_ref(p, a))
    assert st["conflict_free"] == st["rounds"] == 3 * n // 32


def test_cluster_path_rejects_unsupported_shapes(lib):
    p = W.random(1 << 20, 1)
    with pytest.raises(lib.PermError) as e:
        lib.Plan(p, device=False, passes=2)          # 2^20 words do not fit in 16 blocks
    assert e.value.status == -3
    with pytest.raises(lib.PermError):
        lib.Plan(W.random(1 << 16, 1), device=False, passes=2, cluster=3)


@pytest.mark.parametrize("k,fam", [(20, "random"), (20, "bitrev"), (21, "transpose")])
def test_product_tlc_ring_plan_checks_and_runs_on_the_oracle_executor(lib, k, fam):
    # layout 5: TLC passes with 32768-word tiles run through the half-tile ring (the 2^26 /
    # 2^27 structure), schedules in the ring's dense per-round format; exported per tile
    n = 1 << k
    p = W.make_perm(fam, n, seed=k)
    with lib.Plan(p, device=False, layout=5, direct=-1) as pl:
        info = pl.info()
        d = pl.describe()
        kappa, scheds = pl.export()
    assert info["passes"] == 3 and d["layout"] == 5 and info["entry_bits"] == [25, 25, 25]
    r, c, h = info["rows"], info["cols"], tuple(info["h"])
    sched = [s.reshape(-1) for s in scheds]
    assert _ok(OC.check_tlc(p, kappa.astype(np.int64), sched, r, c, h))
    a = W.make_data(n)
    b, st = OT.tlc_apply(a, sched, r, c, h)
    assert np.array_equal(b, OA.apply_ref(p, a))
    assert st["conflict_free"] == st["rounds"] == 3 * n // 32
