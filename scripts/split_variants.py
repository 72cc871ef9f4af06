"""n = 2^30 (L = 32768 lines): half-line ring variants (env PERM_SPLIT read at plan build),
apply time, per-kernel times, sampled parity."""
import json, os, statistics, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
k = int(sys.argv[1]) if len(sys.argv) > 1 else 30
fam = sys.argv[2] if len(sys.argv) > 2 else 'bitrev'
variants = (sys.argv[3] if len(sys.argv) > 3 else 'r1024,k1024,r512,k512').split(',')
n = 1 << k
p = W.make_perm(fam, n)
ha = W.make_data(n)
da = torch.from_numpy(ha.view(np.int32)).cuda(); db = torch.empty_like(da)
idx = np.random.default_rng(1).integers(0, n, size=1 << 22)
for v in variants:
    os.environ['PERM_SPLIT'] = v
    t0 = time.perf_counter(); plan = P.Plan(p); tb = time.perf_counter() - t0
    d = plan.describe()
    ts = []
    for i in range(4):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); plan.apply(da, db); e1.record(); torch.cuda.synchronize()
        if i: ts.append(e0.elapsed_time(e1))
    plan.set_profiling(True); plan.apply(da, db); kt = plan.pass_times(); plan.set_profiling(False)
    b = db.cpu().numpy().view(np.uint32)
    ok = bool(np.array_equal(b[p[idx]], ha[idx]))
    del b
    print(json.dumps({'k': k, 'family': fam, 'variant': v, 'plan_s': tb, 'apply_ms': statistics.median(ts),
                      'kernel_ms': kt, 'threads': [rp['threads'] for rp in d['row_passes']],
                      'dense': [rp['dense'] for rp in d['row_passes']], 'sampled_bitexact': ok}), flush=True)
    plan.close()
