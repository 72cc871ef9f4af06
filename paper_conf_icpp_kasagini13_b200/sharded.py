"""Row-sharded (multi-GPU) apply: libperm steps + all-to-all exchanges.

SURVEY §8e / include/perm.h perm_sharded_step: rank g owns rows
[g*r/G, (g+1)*r/G) of the r x c view (the contiguous shard a[g*n/G:(g+1)*n/G]).
Phases 1 and 3 (row-wise) are local; the column-wise
phase (Lemma 8: transpose, row-wise, transpose) becomes two uniform,
P-independent all-to-all exchanges of n/G^2-element blocks:

    step 0 (R1 + T-pack)  ->  all-to-all  ->  step 1 (R2 + T-pack)  ->  all-to-all  ->  step 2 (R3)

The exchange is torch.distributed.all_to_all_single (NCCL over NVLink/NVSwitch
on GPUs): out chunk i comes from rank i's in chunk for this rank, which is
exactly the block contract of perm_sharded_step. Argument marshalling only —
the data path is libperm's kernels and NCCL.
"""
from __future__ import annotations


class ShardedApply:
    """Apply a row-sharded plan: `steps` provides sharded_step(step, inp, out, stream)
    (a libperm Plan created with world/rank), `exchange(send, recv)` the all-to-all."""

    def __init__(self, steps, exchange=None, group=None):
        self.steps = steps
        self.group = group
        self._exchange = exchange or self._nccl_exchange

    def _nccl_exchange(self, send, recv):
        import torch.distributed as dist
        dist.all_to_all_single(recv, send, group=self.group)

    def __call__(self, a_shard, b_shard, send, recv, stream=None):
        """b_shard <- this rank's rows of b, b[P(i)] = a[i]. send/recv: scratch of n/G elements."""
        self.steps.sharded_step(0, a_shard, send, stream)
        self._exchange(send, recv)
        self.steps.sharded_step(1, recv, send, stream)
        self._exchange(send, recv)
        self.steps.sharded_step(2, recv, b_shard, stream)
        return b_shard


def loopback_exchange(sends, recvs, block: int):
    """All-to-all between G virtual ranks living in one process (one GPU):
    recv_q[g*B:(g+1)*B] = send_g[q*B:(q+1)*B]. Device copies; for tests and single-GPU runs."""
    G = len(sends)
    for g in range(G):
        for q in range(G):
            recvs[q][g * block:(g + 1) * block].copy_(sends[g][q * block:(q + 1) * block])


def apply_virtual(plans, a_shards, b_shards, sends, recvs, stream=None):
    """Run a G-rank sharded apply with all ranks on the current device (plans[g] = rank g)."""
    block = plans[0].info()["block_elems"]
    for g, pl in enumerate(plans):
        pl.sharded_step(0, a_shards[g], sends[g], stream)
    loopback_exchange(sends, recvs, block)
    for g, pl in enumerate(plans):
        pl.sharded_step(1, recvs[g], sends[g], stream)
    loopback_exchange(sends, recvs, block)
    for g, pl in enumerate(plans):
        pl.sharded_step(2, recvs[g], b_shards[g], stream)
    return b_shards
