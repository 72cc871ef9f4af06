"""n = 2^28 / 2^30 single GPU: plan build time, apply time (5-pass), sampled parity
(b[p[i]] == a[i] on 2^22 random i), conventional kernel time."""
import argparse, json, statistics, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
ap = argparse.ArgumentParser()
ap.add_argument('--k', type=int, default=30)
ap.add_argument('--family', default='bitrev')
ap.add_argument('--reps', type=int, default=3)
a = ap.parse_args()
n = 1 << a.k
t0 = time.perf_counter(); p = W.make_perm(a.family, n); tg = time.perf_counter() - t0
ha = W.make_data(n)
t0 = time.perf_counter(); plan = P.Plan(p); tb = time.perf_counter() - t0
info = plan.info()
da = torch.from_numpy(ha.view(np.int32)).cuda(); db = torch.empty_like(da)
def timeit(fn):
    ts = []
    for i in range(a.reps + 1):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 1: ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)
t_apply = timeit(lambda: plan.apply(da, db))
plan.set_profiling(True); plan.apply(da, db); kt = plan.pass_times(); plan.set_profiling(False)
rng = np.random.default_rng(1)
idx = rng.integers(0, n, size=1 << 22)
b = db.cpu().numpy().view(np.uint32)
ok = bool(np.array_equal(b[p[idx]], ha[idx]))
# b must also be a permutation of a's multiset on the sample's image
del b
plan.close()
dp = torch.from_numpy(p).cuda()
t_conv = timeit(lambda: P.scatter_baseline(dp, da, db))
print(json.dumps({'k': a.k, 'family': a.family, 'gen_s': tg, 'plan_s': tb, 'colour_ms': info['build_ms_colour'],
                  'bank_ms': info['build_ms_bank'], 'upload_ms': info['build_ms_upload'], 'passes': info['passes'],
                  'sched_GB': info['sched_bytes'] / 1e9, 'apply_ms': t_apply, 'kernel_ms': kt,
                  'conv_ms': t_conv, 'speedup': t_conv / t_apply,
                  'eff_GBs': 2 * n * 4 / t_apply / 1e6, 'sampled_bitexact': ok, 'sample': 1 << 22}), flush=True)
