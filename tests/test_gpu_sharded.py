"""GPU: the row-sharded path with G virtual ranks on one device, and the whole
sharded apply through libperm's C ABI (perm_apply_sharded: kernels + NCCL).

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
@pytest.mark.parametrize("k", [16, 19, 21, 22])
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


@pytest.mark.parametrize("G", [2, 8])
def test_virtual_ranks_tlc_compact_2pow24(P, G):
    # the row-sharded TLC form with the compact entries that are the default from 2^23 on
    from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
    n = 1 << 24
    shard = n // G
    a = W.make_data(n)
    for fam in ("random", "bitrev"):
        p = W.make_perm(fam, n, seed=G)
        plans = [P.Plan(p, world=G, rank=g) for g in range(G)]
        try:
            info = plans[0].info()
            assert info["passes"] == 3 and max(info["entry_bits"]) < 2 * 13 - 5 + 2, info
            a_sh = [torch.from_numpy(a[g * shard:(g + 1) * shard].view(np.int32).copy()).cuda() for g in range(G)]
            b_sh = [torch.full((shard,), -1, dtype=torch.int32, device="cuda") for _ in range(G)]
            send = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
            recv = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
            apply_virtual(plans, a_sh, b_sh, send, recv)
            torch.cuda.synchronize()
            b = np.concatenate([x.cpu().numpy().view(np.uint32) for x in b_sh])
            assert np.array_equal(b, OA.apply_ref(p, a)), (fam, G)
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


@pytest.mark.parametrize("fam", ["random", "bitrev"])
def test_virtual_ranks_g8_2pow26(P, fam):
    # C3 size with the widest sharding the bench uses (G = 8): default kernels per step
    from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
    G, n = 8, 1 << 26
    shard = n // G
    a = W.make_data(n)
    p = W.make_perm(fam, n, seed=5)
    plans = [P.Plan(p, world=G, rank=g) for g in range(G)]
    try:
        a_sh = [torch.from_numpy(a[g * shard:(g + 1) * shard].view(np.int32).copy()).cuda() for g in range(G)]
        b_sh = [torch.full((shard,), -1, dtype=torch.int32, device="cuda") for _ in range(G)]
        send = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
        recv = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
        apply_virtual(plans, a_sh, b_sh, send, recv)
        torch.cuda.synchronize()
        b = np.concatenate([x.cpu().numpy().view(np.uint32) for x in b_sh])
        assert np.array_equal(b, OA.apply_ref(p, a)), fam
    finally:
        for pl in plans:
            pl.close()


@pytest.mark.parametrize("k", [16, 22])
def test_apply_sharded_through_nccl_world1(P, k):
    # perm_apply_sharded: R1+T-pack, NCCL all-to-all (grouped send/recv on the caller's
    # stream), R2+T-pack, all-to-all, R3 -- all inside libperm. One GPU in this test, so
    # the communicator has one rank (the exchange is NCCL's self send/recv).
    n = 1 << k
    uid = P.nccl_unique_id()
    assert len(uid) == 128
    a = W.make_data(n)
    for fam in ("random", "bitrev", "transpose"):
        p = W.make_perm(fam, n, seed=k)
        with P.Plan(p, world=1, rank=0, nccl_uid=uid if fam == "random" else P.nccl_unique_id()) as pl:
            da = torch.from_numpy(a.view(np.int32).copy()).cuda()
            db = torch.full_like(da, -1)
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                pl.apply_sharded(da, db, s)
            s.synchronize()
            assert np.array_equal(db.cpu().numpy().view(np.uint32), OA.apply_ref(p, a)), fam
            # the exchange alone is the block contract (world 1: a copy)
            x = torch.arange(n, dtype=torch.int32, device="cuda")
            y = torch.zeros_like(x)
            pl.sharded_exchange(x, y)
            torch.cuda.synchronize()
            assert torch.equal(x, y)


def test_apply_sharded_errors(P):
    n = 1 << 16
    p = W.random(n, 3)
    x = torch.zeros(n, dtype=torch.int32, device="cuda")
    y = torch.zeros(n, dtype=torch.int32, device="cuda")
    with P.Plan(p, world=1, rank=0) as pl:                 # no communicator
        with pytest.raises(P.PermError) as ei:
            pl.apply_sharded(x, y)
        assert ei.value.status == -6
        with pytest.raises(P.PermError):
            pl.apply(x, y)                                  # sharded plans: not perm_apply
    with P.Plan(p) as pl:                                   # unsharded plan
        with pytest.raises(P.PermError):
            pl.apply_sharded(x, y)


@pytest.mark.parametrize("G", [2, 4])
@pytest.mark.parametrize("sched_format", [0, -1])
def test_virtual_ranks_half_line_ring(P, G, sched_format):
    # the C4 kernels (lines of 32768 words: the half-line ring, staged dense schedule chunks
    # or re-decoded W64 entries) with segmented column-phase input (one segment per sender),
    # at small n through a wide view (L603): 128 x 32768, rows sharded G ways
    from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
    n = 1 << 22
    shard = n // G
    a = W.make_data(n)
    for fam in ("random", "bitrev"):
        p = W.make_perm(fam, n, seed=G)
        plans = [P.Plan(p, world=G, rank=g, log2c=15, no_tma=-2, sched_format=sched_format) for g in range(G)]
        try:
            d = plans[0].describe()
            assert any(rp["split"] == 1 and rp["L"] == 32768 for rp in d["row_passes"]), d
            a_sh = [torch.from_numpy(a[g * shard:(g + 1) * shard].view(np.int32).copy()).cuda() for g in range(G)]
            b_sh = [torch.full((shard,), -1, dtype=torch.int32, device="cuda") for _ in range(G)]
            send = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
            recv = [torch.empty(shard, dtype=torch.int32, device="cuda") for _ in range(G)]
            apply_virtual(plans, a_sh, b_sh, send, recv)
            torch.cuda.synchronize()
            b = np.concatenate([x.cpu().numpy().view(np.uint32) for x in b_sh])
            assert np.array_equal(b, OA.apply_ref(p, a)), (fam, G, sched_format)
        finally:
            for pl in plans:
                pl.close()
