"""C5 (BASELINE configs[4]; Table II): apply time vs n for every
permutation family with the plan's DEFAULT structure, the conventional D-designated
(L365) and S-designated (L373) kernels on the same inputs, the offline plan-build time
split (colour / bank / upload) and a FULL bit-exact check against numpy's b[p] = a.
Cold L2 (256 MiB write + read before every timed launch). One JSON line per (n, family).

    python scripts/c5_sweep.py --k 16,17,...,30 [--families ...] [--eb 8]
"""
import argparse, json, statistics, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np

ap = argparse.ArgumentParser()
ap.add_argument('--k', default='16,18,20,22,24,26,28')
ap.add_argument('--families', default=','.join(W.FAMILIES))
ap.add_argument('--eb', type=int, default=4)
ap.add_argument('--out', default='')
a = ap.parse_args()
ks = [int(x) for x in a.k.split(',')]
fams = a.families.split(',')
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
peak = json.load(open('MEASURED_PEAKS.json'))['hbm_gbs'] if __import__('os').path.exists('MEASURED_PEAKS.json') else 6539.2
out = open(a.out, 'a') if a.out else None


def timeit(fn, reps):
    ts = []
    for i in range(reps + 3):
        flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.mean(ts), statistics.median(ts), min(ts)


for k in ks:
    n = 1 << k
    host_a = W.make_data(n, elem_bytes=a.eb)
    da = torch.from_numpy(host_a.view(np.int32)).cuda()
    db = torch.empty_like(da)
    reps = max(5, min(50, (1 << 28) // n))
    for fam in fams:
        t0 = time.perf_counter(); p = W.make_perm(fam, n); t_gen = time.perf_counter() - t0
        t0 = time.perf_counter(); plan = P.Plan(p, elem_bytes=a.eb); t_plan = time.perf_counter() - t0
        info, desc = plan.info(), plan.describe()
        apply_mean, apply_med, apply_min = timeit(lambda: plan.apply(da, db), reps)
        ok = bool(np.array_equal(db.cpu().numpy().view(host_a.dtype), scatter_np(p, host_a)))
        sched_bytes = info['sched_bytes']
        plan.close()
        dp = torch.from_numpy(p).cuda()
        conv = timeit(lambda: P.scatter_baseline(dp, da, db, elem_bytes=a.eb), reps)
        dq = torch.from_numpy(inverse_np(p)).cuda()
        gath = timeit(lambda: P.gather_baseline(dq, da, db, elem_bytes=a.eb), reps)
        del dp, dq
        torch.cuda.empty_cache()
        row = {"k": k, "n": n, "eb": a.eb, "family": fam, "p_sha256": W.perm_sha256(p)[:16],
               "passes": info['passes'], "direct": info['direct'], "view": [info['rows'], info['cols']],
               "kernels_per_apply": info['kernels_per_apply'], "gpu_planner": info['gpu_planner'],
               "t_gen_s": t_gen, "t_plan_s": t_plan,
               "t_plan_ms": {"colour": info['build_ms_colour'], "bank": info['build_ms_bank'],
                             "upload": info['build_ms_upload']},
               "sched_bytes": sched_bytes, "D_w_over_n": info['distribution'] / (n * a.eb // 4),
               "apply_us": {"mean": apply_mean, "median": apply_med, "min": apply_min},
               "conv_us": conv[0], "gather_us": gath[0],
               "speedup_vs_conv": conv[0] / apply_mean, "speedup_vs_gather": gath[0] / apply_mean,
               "eff_gbs": 2 * n * a.eb / (apply_mean * 1e-6) / 1e9,
               # read a + write b + the plan's index data (three schedules; q or p for the
               # shortcut kernels; n/32 block indices for the block gather)
               "min_traffic_frac": (2 * n * a.eb + {0: sched_bytes, 1: 4 * n, 2: 4 * n, 3: n // 8}[info['direct']])
                                   / (apply_mean * 1e-6) / 1e9 / peak,
               "bitexact": ok, "reps": reps, "l2": "flushed per launch"}
        line = json.dumps(row)
        print(line, flush=True)
        if out:
            out.write(line + "\n"); out.flush()
    del da, db
    torch.cuda.empty_cache()
