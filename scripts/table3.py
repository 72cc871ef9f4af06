"""Mini Table III (NEXT-3): K uniformly random permutations of
n = 4M: min / avg / max time of the D-designated, S-designated and scheduled
algorithms (cold L2, CUDA events) and D_w(P)/n. The paper used K = 1000 on a GTX-680;
the point is the P-independence of the scheduled time (its spread)."""
import argparse, json, statistics, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
ap = argparse.ArgumentParser()
ap.add_argument('--log2n', type=int, default=22)
ap.add_argument('--perms', type=int, default=32)
ap.add_argument('--reps', type=int, default=5)
a = ap.parse_args()
n = 1 << a.log2n
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
ha = W.make_data(n)
da = torch.from_numpy(ha.view(np.int32)).cuda(); db = torch.empty_like(da)
def timeit(fn):
    ts = []
    for i in range(a.reps + 1):
        flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 1: ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.mean(ts)          # the event clock steps in ~2 us quanta: the mean resolves them
rows = {'D-designated': [], 'S-designated': [], 'scheduled': [], 'D_w/n': []}
for s in range(a.perms):
    p = W.random(n, 42 + s)
    dp = torch.from_numpy(p).cuda(); dq = torch.from_numpy(inverse_np(p)).cuda()
    rows['D-designated'].append(timeit(lambda: P.scatter_baseline(dp, da, db)))
    rows['S-designated'].append(timeit(lambda: P.gather_baseline(dq, da, db)))
    with P.Plan(p) as plan:
        dw = plan.info()['distribution']          # D_w(P), the planner's count (L389-L401)
        rows['scheduled'].append(timeit(lambda: plan.apply(da, db)))
        if s == 0:
            ok = bool(np.array_equal(db.cpu().numpy().view(np.uint32), scatter_np(p, ha)))
    rows['D_w/n'].append(dw / n)
out = {k: {'min': min(v), 'avg': statistics.mean(v), 'max': max(v)} for k, v in rows.items()}
out['n'] = n; out['perms'] = a.perms; out['unit'] = 'us (D_w/n: ratio)'; out['bitexact_first'] = ok
print(json.dumps(out))
