"""Apply time vs n for several plan options and the conventional kernels (cold L2).
Prints one JSON line per (n, family, config). Plan-build time included."""
import argparse, json, statistics, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
ap = argparse.ArgumentParser()
ap.add_argument('--k', default='22,24,25,26')
ap.add_argument('--families', default='random')
ap.add_argument('--configs', default='[{}]')
ap.add_argument('--reps', type=int, default=10)
ap.add_argument('--check', action='store_true')
a = ap.parse_args()
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
def timeit(fn, reps):
    ts = []
    for i in range(reps + 2):
        flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)
for k in [int(x) for x in a.k.split(',')]:
    n = 1 << k
    reps = max(3, min(a.reps, (1 << 28) // n))
    ha = W.make_data(n)
    da = torch.from_numpy(ha.view(np.int32)).cuda(); db = torch.empty_like(da)
    for fam in a.families.split(','):
        p = W.make_perm(fam, n)
        dp = torch.from_numpy(p).cuda()
        conv = timeit(lambda: P.scatter_baseline(dp, da, db), reps)
        del dp
        ref = scatter_np(p, ha) if a.check else None
        for cfg in json.loads(a.configs):
            kw = dict(cfg)
            if 'h' in kw: kw['h'] = tuple(kw['h'])
            try:
                t0 = time.perf_counter(); plan = P.Plan(p, **kw); tb = time.perf_counter() - t0
                info = plan.info()
                t = timeit(lambda: plan.apply(da, db), reps)
                ok = None
                if a.check:
                    ok = bool(np.array_equal(db.cpu().numpy().view(np.uint32), ref))
                print(json.dumps({'k': k, 'family': fam, 'cfg': cfg, 'passes': info['passes'],
                                  'layout': plan.describe().get('layout'), 'apply_us': t, 'conv_us': conv,
                                  'speedup': conv / t, 'eff_gbs': 2 * n * 4 / t / 1e3,
                                  'plan_s': tb, 'colour_ms': info['build_ms_colour'], 'bank_ms': info['build_ms_bank'],
                                  'sched_MB': info['sched_bytes'] / 1e6, 'ok': ok}), flush=True)
                plan.close()
            except Exception as e:
                print(json.dumps({'k': k, 'family': fam, 'cfg': cfg, 'error': str(e)}), flush=True)
