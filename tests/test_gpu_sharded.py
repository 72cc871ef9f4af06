"""GPU: the row-sharded path with G virtual ranks on one device.

Every rank's perm_sharded_step kernels run for real (R1+T-pack, R2 over G segments
per column + T-pack, R3 over G segments per row); the all-to-all between steps is
a device loopback (paper_conf_icpp_kasagini13_b200.sharded.loopback_exchange) —
the same block contract NCCL's all_to_all_single fulfils across GPUs. The
concatenated b shards must equal the oracle's b bit for bit.
"""
import numpy as np
import pytest

import workloads as W
from oracle import apply as OA

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


@pytest.mark.parametrize("no_tma", [0, 1, -1, -2])
@pytest.mark.parametrize("G", [1, 2, 4, 8])
@pytest.mark.parametrize("k", [16, 19, 22])
def test_virtual_ranks(P, G, k, no_tma):
    from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
    n = 1 << k
    shard = n // G
    a = W.make_data(n)
    for fam in ("random", "bitrev", "transpose"):
        p = W.make_perm(fam, n, seed=G + k)
        # dense schedule bitstreams with the SG kernels (no_tma = -1)
        fmt = 2 if no_tma == -1 else 0
        plans = [P.Plan(p, world=G, rank=g, no_tma=no_tma, sched_format=fmt) for g in range(G)]
        try:
            a_sh = [torch.from_numpy(a[g * shard:(g + 1) * shard].view(np.int32).copy()).cuda() for g in range(G)]
            b_sh = [torch.full((shard,), -1, dtype=torch.int32, device="cuda") for _ in range(G)]
            send = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
            recv = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
            apply_virtual(plans, a_sh, b_sh, send, recv)
            torch.cuda.synchronize()
            b = np.concatenate([x.cpu().numpy().view(np.uint32) for x in b_sh])
            assert np.array_equal(b, OA.apply_ref(p, a)), (fam, G, k)
        finally:
            for pl in plans:
                pl.close()


def test_sharded_step_errors(P):
    n = 1 << 16
    with P.Plan(W.random(n, 1), world=2, rank=0) as pl:
        x = torch.zeros(n, dtype=torch.int32, device="cuda")
        with pytest.raises(P.PermError):
            pl.sharded_step(3, x, x[n // 2:])
        with pytest.raises(P.PermError):
            pl.sharded_step(0, x, x)
    with P.Plan(W.random(n, 1)) as pl:          # unsharded plan
        x = torch.zeros(n, dtype=torch.int32, device="cuda")
        y = torch.zeros(n, dtype=torch.int32, device="cuda")
        with pytest.raises(P.PermError):
            pl.sharded_step(0, x, y)
