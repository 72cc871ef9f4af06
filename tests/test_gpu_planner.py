"""GPU planner (gplan.cu): the row-level and bank-level
colourings computed on the device must pass the oracle's independent plan
checker (oracle/check.py: PAPER.md L537 (1)-(2), L519, L531-L533) and drive
perm_apply to b[P(i)] = a[i] bit-exactly (L361)."""
import numpy as np
import pytest

import workloads as W
from oracle import apply as OA
from oracle import check as OC

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_kasagini13_b200 import build
    build.build()
    import paper_conf_icpp_kasagini13_b200 as pkg
    return pkg


def decode(sched):
    s = np.asarray(sched, dtype=np.uint32)
    return (s >> 16).astype(np.int64), (s & 0xFFFF).astype(np.int64)


def apply_ok(P, plan, p, a):
    da = torch.from_numpy(a.view(np.int32)).cuda()
    db = torch.full_like(da, -1)
    plan.apply(da, db)
    torch.cuda.synchronize()
    return np.array_equal(db.cpu().numpy().view(np.uint32), OA.apply_ref(p, a))


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [10, 12, 13, 16, 19])
def test_gpu_planner_line_schedules(P, fam, k):
    # per-line (W64) schedules: 5-pass / fused structures
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm(fam, n, seed=100 + k)
    passes = 1 if k <= 14 and k % 2 == 0 else 5
    # 5-pass: also the dense bitstream format (device-side packing of both formats)
    for fmt in ((0,) if passes == 1 else (0, 2)):
        with P.Plan(p, passes=passes, gpu_planner=1, direct=-1, sched_format=fmt) as plan:
            info = plan.info()
            assert info["gpu_planner"] == 1
            kappa, scheds = plan.export()
            OC.assert_plan(p, kappa.astype(np.int64), [decode(s) for s in scheds], r, c, 32)
            assert apply_ok(P, plan, p, W.make_data(n))


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [16, 18, 20, 22])
def test_gpu_planner_tlc(P, fam, k):
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm(fam, n, seed=200 + k)
    with P.Plan(p, passes=3, layout=3, gpu_planner=1, direct=-1) as plan:
        info = plan.info()
        assert info["gpu_planner"] == 1
        kappa, scheds = plan.export()
        res = OC.check_tlc(p, kappa.astype(np.int64), [s.reshape(-1) for s in scheds], r, c,
                           tuple(info["h"]))
        assert all(res.values()), res
        assert apply_ok(P, plan, p, W.make_data(n))


def test_gpu_planner_is_default_for_device_plans(P):
    n = 1 << 20
    p = W.random(n, 5)
    with P.Plan(p) as plan:
        assert plan.info()["gpu_planner"] == 1
    with P.Plan(p, gpu_planner=-1) as plan:
        assert plan.info()["gpu_planner"] == 0
    with P.Plan(W.random(1 << 16, 5)) as plan:       # small n: host threads
        assert plan.info()["gpu_planner"] == 0


def test_gpu_planner_2pow26_and_fp64(P):
    # BASELINE configs[2] size through the GPU planner (5-pass per-line schedules),
    # and 8-byte elements (word pairs, Table II(b))
    n = 1 << 26
    p = W.random(n, 42)
    a = W.make_data(n)
    with P.Plan(p, gpu_planner=1) as plan:
        assert plan.info()["passes"] == 5
        assert apply_ok(P, plan, p, a)
    n8 = 1 << 20
    p8 = W.random(n8, 3)
    a8 = W.make_data(n8, elem_bytes=8)
    with P.Plan(p8, elem_bytes=8, gpu_planner=1) as plan:
        da = torch.from_numpy(a8.view(np.int64)).cuda()
        db = torch.empty_like(da)
        plan.apply(da, db)
        torch.cuda.synchronize()
        assert np.array_equal(db.cpu().numpy().view(np.uint64), OA.apply_ref(p8, a8))
