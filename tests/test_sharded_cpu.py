"""Row-sharded path without GPUs.

The C++ planner builds each rank's sharded plan on the CPU (perm_plan_create_sharded_host);
a numpy stand-in executes perm_sharded_step exactly as include/perm.h specifies it (R = the
per-line permutation of the exported (sigma, t) schedule, T = transpose, block layouts of
the all-to-all); the Python driver paper_conf_icpp_kasagini13_b200/sharded.py runs the
steps with a real torch.distributed all-to-all over gloo (world_size 2, two processes) and
in-process (G = 4, 8 virtual ranks). Every rank's b shard must equal the oracle's slice.
"""
import os
import socket

import numpy as np
import pytest
import torch

import workloads as W
from oracle import apply as OA


def _lib():
    from paper_conf_icpp_kasagini13_b200 import build
    build.build()
    import paper_conf_icpp_kasagini13_b200 as P
    return P


class FakeSteps:
    """numpy execution of perm_sharded_step for the per-line (5-pass) form
    (test infrastructure, not the product)."""

    def __init__(self, p, G, g):
        P = _lib()
        with P.Plan(p, device=False, world=G, rank=g, passes=5) as pl:
            info = pl.info()
            _, sched = pl.export()
        self.r, self.c = info["rows"], info["cols"]
        self.G = G
        self.rl, self.cl = self.r // G, self.c // G
        self.src, self.dst = [], []
        for s in sched:
            s = s.astype(np.int64)
            L = s.shape[1]
            lane = np.arange(L, dtype=np.int64)[None, :] % 32
            self.src.append(32 * (s >> 16) + lane)
            self.dst.append(s & 0xFFFF)

    def _permute(self, X, f):
        out = np.empty_like(X)
        rows = np.arange(X.shape[0])[:, None]
        out[rows, self.dst[f]] = X[rows, self.src[f]]
        return out

    def sharded_step(self, step, inp, out, stream=None):
        x = inp.numpy().view(np.uint32)
        G, r, c, rl, cl = self.G, self.r, self.c, self.rl, self.cl
        if step == 0:
            Y = self._permute(x.reshape(rl, c), 0)                        # R1 on my rows
            res = Y.T                                                      # T-pack (c x rl)
        elif step == 1:
            X = x.reshape(G, cl, rl).transpose(1, 0, 2).reshape(cl, r)    # segments -> columns
            res = self._permute(X, 1).T                                    # R2, T-pack (r x cl)
        else:
            X = x.reshape(G, rl, cl).transpose(1, 0, 2).reshape(rl, c)    # segments -> rows
            res = self._permute(X, 2)                                      # R3 -> b rows
        out.numpy().view(np.uint32)[:] = np.ascontiguousarray(res).reshape(-1)
        return out


class FakeTlcSteps:
    """numpy execution of perm_sharded_step for the TLC form: the rank's
    exported tile entries (src << 16 | dst) applied tile by tile; tiles of passes 2 and 3
    gathered as one segment per sender; outputs scattered as chunks into the per-peer X1 /
    X2 layouts (single-GPU layouts with r -> r/G, c -> c/G). Test infrastructure."""

    def __init__(self, p, G, g):
        P = _lib()
        with P.Plan(p, device=False, world=G, rank=g) as pl:
            info = pl.info()
            d = pl.describe()
            _, sched = pl.export()
        assert d["layout"] == 3 and info["passes"] == 3
        self.r, self.c = info["rows"], info["cols"]
        self.G = G
        self.h = [t["h"] for t in d["tlc"]]
        self.sched = [np.asarray(x, dtype=np.int64).reshape(-1) for x in sched]

    def _tiles(self, f, tiles, HL):
        e = self.sched[f].reshape(len(tiles), HL)
        src, dst = e >> 16, e & 0xFFFF
        out = []
        for T, A in enumerate(tiles):
            B = np.empty_like(A)
            B[dst[T]] = A[src[T]]
            out.append(B)
        return out

    def sharded_step(self, step, inp, out, stream=None):
        x = inp.numpy().view(np.uint32)
        y = out.numpy().view(np.uint32)
        G, r, c = self.G, self.r, self.c
        rl, cl = r // G, c // G
        h1, h2, h3 = self.h
        Bw = rl * cl
        if step == 0:
            HL = h1 * c
            tiles = [x[T * HL:(T + 1) * HL] for T in range(rl // h1)]
            cw, cs = h1 * h2, rl * h2
            for T, B in enumerate(self._tiles(0, tiles, HL)):
                for m in range(c // h2):
                    y[m * cs + T * cw:m * cs + (T + 1) * cw] = B[m * cw:(m + 1) * cw]
        elif step == 1:
            sl, HL = rl * h2, r * h2
            tiles = [np.concatenate([x[q * Bw + K * sl:q * Bw + (K + 1) * sl] for q in range(G)])
                     for K in range(cl // h2)]
            cw, cs = h3 * h2, cl * h3
            for K, B in enumerate(self._tiles(1, tiles, HL)):
                for m in range(r // h3):
                    y[m * cs + K * cw:m * cs + (K + 1) * cw] = B[m * cw:(m + 1) * cw]
        else:
            sl, HL = cl * h3, h3 * c
            tiles = [np.concatenate([x[q * Bw + I * sl:q * Bw + (I + 1) * sl] for q in range(G)])
                     for I in range(rl // h3)]
            for I, B in enumerate(self._tiles(2, tiles, HL)):
                y[I * HL:(I + 1) * HL] = B
        return out


@pytest.mark.parametrize("G", [1, 2, 4, 8])
@pytest.mark.parametrize("fam", ["random", "bitrev", "transpose"])
def test_virtual_ranks_tlc_form_numpy(G, fam):
    from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
    n = 1 << 16
    p = W.make_perm(fam, n, seed=G + 1)
    a = W.make_data(n)
    shard = n // G
    steps = [FakeTlcSteps(p, G, g) for g in range(G)]

    class Wrap:
        def __init__(self, s):
            self.s = s

        def info(self):
            return {"block_elems": n // (G * G)}

        def sharded_step(self, *args):
            return self.s.sharded_step(*args)

    a_sh = [torch.from_numpy(a[g * shard:(g + 1) * shard].view(np.int32).copy()) for g in range(G)]
    b_sh = [torch.empty(shard, dtype=torch.int32) for _ in range(G)]
    send = [torch.empty(shard, dtype=torch.int32) for _ in range(G)]
    recv = [torch.empty(shard, dtype=torch.int32) for _ in range(G)]
    apply_virtual([Wrap(s) for s in steps], a_sh, b_sh, send, recv)
    b = np.concatenate([x.numpy().view(np.uint32) for x in b_sh])
    assert np.array_equal(b, OA.apply_ref(p, a))


@pytest.mark.parametrize("G", [1, 2, 4, 8])
@pytest.mark.parametrize("fam", ["random", "bitrev", "transpose"])
def test_virtual_ranks_numpy(G, fam):
    from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
    n = 1 << 16
    p = W.make_perm(fam, n, seed=G)
    a = W.make_data(n)
    shard = n // G
    steps = [FakeSteps(p, G, g) for g in range(G)]

    class Wrap:
        def __init__(self, s):
            self.s = s

        def info(self):
            return {"block_elems": n // (G * G)}

        def sharded_step(self, *args):
            return self.s.sharded_step(*args)

    a_sh = [torch.from_numpy(a[g * shard:(g + 1) * shard].view(np.int32).copy()) for g in range(G)]
    b_sh = [torch.empty(shard, dtype=torch.int32) for _ in range(G)]
    send = [torch.empty(shard, dtype=torch.int32) for _ in range(G)]
    recv = [torch.empty(shard, dtype=torch.int32) for _ in range(G)]
    apply_virtual([Wrap(s) for s in steps], a_sh, b_sh, send, recv)
    b = np.concatenate([x.numpy().view(np.uint32) for x in b_sh])
    assert np.array_equal(b, OA.apply_ref(p, a))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _gloo_worker(rank, world, port, k, fam, q, tlc=False):
    import torch.distributed as dist
    from paper_conf_icpp_kasagini13_b200.sharded import ShardedApply
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n = 1 << k
        p = W.make_perm(fam, n, seed=11)
        a = W.make_data(n)
        shard = n // world
        steps = (FakeTlcSteps if tlc else FakeSteps)(p, world, rank)
        run = ShardedApply(steps)            # exchange = torch.distributed.all_to_all_single
        a_sh = torch.from_numpy(a[rank * shard:(rank + 1) * shard].view(np.int32).copy())
        b_sh = torch.empty(shard, dtype=torch.int32)
        send = torch.empty(shard, dtype=torch.int32)
        recv = torch.empty(shard, dtype=torch.int32)
        run(a_sh, b_sh, send, recv)
        ref = OA.apply_ref(p, a)[rank * shard:(rank + 1) * shard]
        q.put((rank, bool(np.array_equal(b_sh.numpy().view(np.uint32), ref))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("tlc", [False, True])
@pytest.mark.parametrize("fam", ["random", "bitrev"])
def test_gloo_world2(fam, tlc):
    import torch.multiprocessing as mp
    _lib()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, 16, fam, q, tlc)) for r in range(2)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(timeout=300)
    results = dict(q.get(timeout=10) for _ in range(2))
    assert results == {0: True, 1: True}


def test_sharded_plan_info_and_errors():
    P = _lib()
    n = 1 << 16
    p = W.random(n, 1)
    with P.Plan(p, device=False, world=4, rank=3) as pl:
        inf = pl.info()
        assert (inf["world"], inf["rank"], inf["shard_elems"], inf["block_elems"]) == (4, 3, n // 4, n // 16)
    with pytest.raises(P.PermError):
        P.Plan(p, device=False, world=3, rank=0)           # not a power of two
    with pytest.raises(P.PermError):
        P.Plan(p, device=False, world=16, rank=0)          # r/world < 32 (256 x 256 view)
