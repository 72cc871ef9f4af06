"""Row-sharded (multi-GPU) apply: marshalling around libperm's sharded C ABI.

SURVEY §8e / include/perm.h: rank g owns rows [g*r/G, (g+1)*r/G) of the r x c
view (the contiguous shard a[g*n/G:(g+1)*n/G]). Phases 1 and 3 (row-wise,
PAPER.md L537-L539) are local; the column-wise phase (Lemma 8: transpose,
row-wise, transpose) becomes two uniform, P-independent all-to-all exchanges of
n/G^2-element blocks:

    step 0 (R1 + T-pack)  ->  all-to-all  ->  step 1 (R2 + T-pack)  ->  all-to-all  ->  step 2 (R3)

Product path: ``sharded_plan(p, group)`` makes the ncclUniqueId on rank 0,
broadcasts its bytes over the torch.distributed group and creates the plan with
it; ``plan.apply_sharded(a_shard, b_shard)`` then runs all five stages inside
libperm (kernels + NCCL send/recv on the caller's stream).

``ShardedApply`` drives the same steps with a caller-supplied exchange
(torch.distributed.all_to_all_single; gloo in the CPU tests) and
``apply_virtual`` runs G ranks on one device with loopback copies (tests).
"""
from __future__ import annotations


def sharded_plan(p, group=None, **kw):
    """Rank `dist.get_rank(group)` of a `dist.get_world_size(group)`-rank sharded plan with
    an NCCL communicator (collective: every rank of the group must call it)."""
    import torch
    import torch.distributed as dist
    from . import _lib
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    uid = _lib.nccl_unique_id() if rank == 0 else bytes(128)
    buf = torch.tensor(list(uid), dtype=torch.uint8)
    if dist.get_backend(group) == "nccl":
        buf = buf.cuda()
    dist.broadcast(buf, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    uid = bytes(buf.cpu().tolist())
    return _lib.Plan(p, world=world, rank=rank, nccl_uid=uid, **kw)


class ShardedApply:
    """Apply a row-sharded plan: `steps` provides sharded_step(step, inp, out, stream)
    (a libperm Plan created with world/rank), `exchange(send, recv)` the all-to-all."""

    def __init__(self, steps, exchange=None, group=None):
        self.steps = steps
        self.group = group
        self._exchange = exchange or self._dist_exchange

    def _dist_exchange(self, send, recv):
        import torch.distributed as dist
        dist.all_to_all_single(recv, send, group=self.group)

    def _exchange_on(self, stream, send, recv):
        # the exchange is issued on the stream the steps run on (torch.distributed uses
        # the current stream), so the steps and the exchange stay ordered
        if stream is not None and not isinstance(stream, int) and hasattr(stream, "cuda_stream"):
            import torch
            with torch.cuda.stream(stream):
                self._exchange(send, recv)
        else:
            self._exchange(send, recv)

    def __call__(self, a_shard, b_shard, send, recv, stream=None):
        """b_shard <- this rank's rows of b, b[P(i)] = a[i]. send/recv: scratch of n/G elements."""
        self.steps.sharded_step(0, a_shard, send, stream)
        self._exchange_on(stream, send, recv)
        self.steps.sharded_step(1, recv, send, stream)
        self._exchange_on(stream, send, recv)
        self.steps.sharded_step(2, recv, b_shard, stream)
        return b_shard


def loopback_exchange(sends, recvs, block: int):
    """All-to-all between G virtual ranks living in one process (one GPU):
    recv_q[g*B:(g+1)*B] = send_g[q*B:(q+1)*B]. Device copies on the current stream."""
    G = len(sends)
    for g in range(G):
        for q in range(G):
            recvs[q][g * block:(g + 1) * block].copy_(sends[g][q * block:(q + 1) * block])


def apply_virtual(plans, a_shards, b_shards, sends, recvs, stream=None):
    """Run a G-rank sharded apply with all ranks on the current device (plans[g] = rank g).
    The steps run on `stream` (default: the current stream), the loopback copies too."""
    import contextlib
    block = plans[0].info()["block_elems"]
    ctx = contextlib.nullcontext()
    if stream is not None and hasattr(stream, "cuda_stream"):
        import torch
        ctx = torch.cuda.stream(stream)
    with ctx:
        for g, pl in enumerate(plans):
            pl.sharded_step(0, a_shards[g], sends[g], stream)
        loopback_exchange(sends, recvs, block)
        for g, pl in enumerate(plans):
            pl.sharded_step(1, recvs[g], sends[g], stream)
        loopback_exchange(sends, recvs, block)
        for g, pl in enumerate(plans):
            pl.sharded_step(2, recvs[g], b_shards[g], stream)
    return b_shards
