"""Per-block phase timeline of the single-launch cluster path (globaltimer stamps), cold L2:
start / a landed / phase 1 done / barrier A / exchange 1 landed / phase 2 done / barrier B /
exchange 2 landed / phase 3 done (store issued) / store read / exit, relative to the first
block's start; min / median / max over the cluster's blocks, median over 20 applies."""
import argparse, json, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
ap = argparse.ArgumentParser()
ap.add_argument('--log2n', type=int, default=16)
ap.add_argument('--cfg', default='{}')
a = ap.parse_args()
n = 1 << a.log2n
plan = P.Plan(W.random(n, 42), **json.loads(a.cfg))
d = plan.describe()
assert d['passes'] == 2, d
C = d.get('cluster')
da = torch.from_numpy(W.make_data(n).view(np.int32)).cuda(); db = torch.empty_like(da)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
plan.set_tracing(True)
names = ['start', 'a_landed', 'phase1', 'barA', 'x1_landed', 'phase2', 'barB', 'x2_landed', 'phase3', 'store_read', 'exit']
runs = []
for i in range(23):
    flush.zero_(); flush.sum(); plan.apply(da, db); torch.cuda.synchronize()
    if i < 3:
        continue
    tr = plan.trace().astype(np.int64)[0][:C, :11]
    t0 = tr[:, 0].min()
    runs.append((tr - t0) / 1e3)
r = np.stack(runs)                      # [run][block][slot]
print(f"n=2^{a.log2n} cluster={C}")
for s, nm in enumerate(names):
    col = r[:, :, s]
    print(f"  {nm:>11}: min {np.median(col.min(1)):6.2f}  med {np.median(np.median(col, 1)):6.2f}  max {np.median(col.max(1)):6.2f}")
