"""One plan, a few applies: small enough to run under ncu (1 GPU)."""
import argparse, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
ap = argparse.ArgumentParser()
ap.add_argument('--log2n', type=int, default=22)
ap.add_argument('--family', default='random')
ap.add_argument('--passes', type=int, default=0)
ap.add_argument('--h', default='0,0,0')
ap.add_argument('--reps', type=int, default=3)
ap.add_argument('--layout', type=int, default=0)
ap.add_argument('--stages', type=int, default=0)
ap.add_argument('--fuse', type=int, default=0)
ap.add_argument('--log2c', type=int, default=0)
ap.add_argument('--baseline', action='store_true')
a = ap.parse_args()
n = 1 << a.log2n
p = W.make_perm(a.family, n)
plan = P.Plan(p, passes=a.passes, h=tuple(int(x) for x in a.h.split(',')), layout=a.layout, stages=a.stages, fuse=a.fuse, log2c=a.log2c)
da = torch.from_numpy(W.make_data(n).view(np.int32)).cuda(); db = torch.empty_like(da)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
dp = torch.from_numpy(p).cuda()
for _ in range(a.reps):
    flush.zero_(); flush.sum()
    plan.apply(da, db)
    if a.baseline:
        flush.zero_()
        P.scatter_baseline(dp, da, db)
torch.cuda.synchronize()
print(plan.describe())
