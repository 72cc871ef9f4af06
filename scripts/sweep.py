"""Time perm_apply for several plan options (cold L2), plus the scatter baseline."""
import argparse, json, statistics, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
ap = argparse.ArgumentParser()
ap.add_argument('--log2n', type=int, default=22)
ap.add_argument('--family', default='random')
ap.add_argument('--configs', default='[{}]')
ap.add_argument('--reps', type=int, default=20)
ap.add_argument('--check', action='store_true')
ap.add_argument('--warm', action='store_true')
a = ap.parse_args()
n = 1 << a.log2n
p = W.make_perm(a.family, n)
host_a = W.make_data(n)
da = torch.from_numpy(host_a.view(np.int32)).cuda(); db = torch.empty_like(da)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
ref = scatter_np(p, host_a) if a.check else None
def timeit(fn):
    ts = []
    for i in range(a.reps + 3):
        if not a.warm: flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
    # mean: the event clock of this box steps in ~2 us quanta (the mean resolves below one step)
    return statistics.mean(ts), min(ts)
dp = torch.from_numpy(p).cuda()
med, mn = timeit(lambda: P.scatter_baseline(dp, da, db))
print(json.dumps({'n': n, 'family': a.family, 'kernel': 'scatter', 'us_med': med, 'us_min': mn}), flush=True)
for cfg in json.loads(a.configs):
    try:
        kw = dict(cfg)
        if 'h' in kw: kw['h'] = tuple(kw['h'])
        use_graph = kw.pop('graph', False)
        plan = P.Plan(p, **kw)
        if use_graph:
            st = torch.cuda.Stream()
            plan.apply(da, db); torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=st):
                plan.apply(da, db, stream=st)
            med, mn = timeit(lambda: g.replay())
        else:
            med, mn = timeit(lambda: plan.apply(da, db))
        ok = None
        if a.check:
            ok = bool(np.array_equal(db.cpu().numpy().view(np.uint32), ref))
        plan.set_profiling(True)
        ks = []
        for _ in range(5):
            if not a.warm: flush.zero_(); flush.sum()
            plan.apply(da, db); ks.append(plan.pass_times())
        plan.set_profiling(False)
        kmed = [statistics.median(x[i] * 1e3 for x in ks) for i in range(len(ks[0]))]
        d = plan.describe()
        print(json.dumps({'cfg': cfg, 'us_med': med, 'us_min': mn, 'ok': ok, 'kernels_us': kmed,
                          'grid': [rp.get('grid') for rp in d.get('row_passes', [])],
                          'ept': [rp.get('ept') for rp in d.get('row_passes', [])]}), flush=True)
        plan.close()
    except Exception as e:
        print(json.dumps({'cfg': cfg, 'error': str(e)}), flush=True)
