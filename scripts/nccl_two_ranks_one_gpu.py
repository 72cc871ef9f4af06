"""Probe: two ranks of perm_apply_sharded on ONE GPU (both ranks on cuda:0), NCCL exchange.
NCCL normally refuses two ranks on one device; this records whether it does here.

    python -m torch.distributed.run --nproc-per-node 2 --master-addr 127.0.0.1 \
        --master-port 29561 scripts/nccl_two_ranks_one_gpu.py
"""
import os, sys
import numpy as np
import torch
import torch.distributed as dist
sys.path.insert(0, '.')
import workloads as W
from paper_conf_icpp_kasagini13_b200 import _lib
from paper_conf_icpp_kasagini13_b200.sharded import sharded_plan

rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dist.init_process_group("gloo", rank=rank, world_size=world)
n = 1 << 20
p = W.random(n, 3)
a = W.make_data(n)
shard = n // world
try:
    pl = sharded_plan(p)
    da = torch.from_numpy(a[rank * shard:(rank + 1) * shard].view(np.int32).copy()).cuda()
    db = torch.full_like(da, -1)
    pl.apply_sharded(da, db)
    torch.cuda.synchronize()
    ref = np.empty_like(a)
    ref[p] = a
    ok = np.array_equal(db.cpu().numpy().view(np.uint32), ref[rank * shard:(rank + 1) * shard])
    print(f"rank {rank}: perm_apply_sharded world {world} on one GPU: {'bit-exact' if ok else 'MISMATCH'}", flush=True)
    pl.close()
except _lib.PermError as e:
    print(f"rank {rank}: {e}", flush=True)
dist.destroy_process_group()
