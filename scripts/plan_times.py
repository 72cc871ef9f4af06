"""Plan-build (offline) time: host planner vs GPU planner, per
n and family, with a sampled bit-exact apply check of the GPU-planned plan.
    python scripts/plan_times.py 20,22,24,26 random,bitrev [host]
"""
import json, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P

ks = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else '20,22,24').split(',')]
fams = (sys.argv[2] if len(sys.argv) > 2 else 'random').split(',')
with_host = len(sys.argv) > 3 and sys.argv[3] == 'host'
for k in ks:
    n = 1 << k
    a = W.make_data(n)
    for fam in fams:
        p = W.make_perm(fam, n)
        rec = {'k': k, 'family': fam}
        for name, gp in (('gpu', 1), ('host', -1)):
            if name == 'host' and not with_host:
                continue
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            plan = P.Plan(p, gpu_planner=gp, direct=-1)
            dt = time.perf_counter() - t0
            info = plan.info()
            rec[name] = {'plan_s': dt, 'colour_ms': info['build_ms_colour'], 'bank_ms': info['build_ms_bank'],
                         'upload_ms': info['build_ms_upload'], 'gpu_planner': info['gpu_planner'],
                         'threads': info['planner_threads']}
            if name == 'gpu':
                da = torch.from_numpy(a.view(np.int32)).cuda(); db = torch.empty_like(da)
                plan.apply(da, db); torch.cuda.synchronize()
                b = db.cpu().numpy().view(np.uint32)
                idx = np.random.default_rng(k).integers(0, n, size=min(n, 1 << 22))
                rec['gpu']['sampled_bitexact'] = bool(np.array_equal(b[p[idx]], a[idx]))
                del da, db
            plan.close()
        print(json.dumps(rec), flush=True)
