"""Small-n regime (NEXT-4, PAPER.md L129 / L701 crossover): apply time of the cluster path
(one launch, DSMEM exchanges), the three-launch TLC path, its single-launch variant
(fuse=1) and the conventional D-/S-designated kernels, cold L2, bit-exact checked.
    python scripts/small_n.py [k,...] [fam,...]
"""
import json, statistics, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np

ks = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "15,16,17,18,19,20,21").split(",")]
fams = (sys.argv[2] if len(sys.argv) > 2 else "random,bitrev,transpose").split(",")
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
REPS = 60


def timeit(fn):
    ts = []
    for i in range(REPS + 3):
        flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
    # the event clock of this box steps in ~2.05 us quanta: the mean over many cold
    # repetitions (which dither across the steps) resolves below one step, the median does not
    return statistics.mean(ts), min(ts)


for k in ks:
    n = 1 << k
    ha = W.make_data(n)
    da = torch.from_numpy(ha.view(np.int32)).cuda(); db = torch.empty_like(da)
    for fam in fams:
        p = W.make_perm(fam, n)
        ref = scatter_np(p, ha)
        dp = torch.from_numpy(p).cuda(); dq = torch.from_numpy(inverse_np(p)).cuda()
        row = {"k": k, "family": fam}
        row["scatter_us"] = timeit(lambda: P.scatter_baseline(dp, da, db))[0]
        row["gather_us"] = timeit(lambda: P.gather_baseline(dq, da, db))[0]
        cfgs = {"tlc3": dict(passes=3, layout=3), "tlc_fused": dict(passes=3, layout=3, fuse=1),
                "cluster8": dict(passes=2, cluster=8), "cluster16": dict(passes=2, cluster=16),
                "cluster4": dict(passes=2, cluster=4)}
        for name, kw in cfgs.items():
            try:
                with P.Plan(p, direct=-1, **kw) as plan:
                    med, mn = timeit(lambda: plan.apply(da, db))
                    ok = bool(np.array_equal(db.cpu().numpy().view(np.uint32), ref))
                row[name + "_us"] = med
                row[name + "_min_us"] = mn
                row[name + "_ok"] = ok
            except P.PermError as e:
                row[name + "_err"] = str(e)[:60]
        print(json.dumps(row), flush=True)
