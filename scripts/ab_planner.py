"""A/B: apply time of host-planned vs GPU-planned schedules for the same P (cold L2)."""
import json, statistics, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
k = int(sys.argv[1]) if len(sys.argv) > 1 else 22
fams = (sys.argv[2] if len(sys.argv) > 2 else 'random,bitrev').split(',')
n = 1 << k
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
a = torch.from_numpy(W.make_data(n).view(np.int32)).cuda(); b = torch.empty_like(a)
for fam in fams:
    p = W.make_perm(fam, n)
    plans = {'host': P.Plan(p, gpu_planner=-1, direct=-1), 'gpu': P.Plan(p, gpu_planner=1, direct=-1)}
    ts = {kk: [] for kk in plans}
    for it in range(60):
        for kk, pl in plans.items():
            flush.zero_(); flush.sum()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); pl.apply(a, b); e1.record(); torch.cuda.synchronize()
            if it >= 5: ts[kk].append(e0.elapsed_time(e1) * 1e3)
    print(json.dumps({'k': k, 'family': fam, **{kk: statistics.median(v) for kk, v in ts.items()},
                      **{kk + '_min': min(v) for kk, v in ts.items()}}), flush=True)
    for pl in plans.values(): pl.close()
