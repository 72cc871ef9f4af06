"""How the L2-flush recipe shapes a cold apply: event-timed perm_apply (n = 2^22 random)
and the median landing time of pass 1's first tile (globaltimer trace) after
  rw     : zero_ + sum of a 256 MiB buffer (bench.py's flush)
  rw_r   : zero_ + sum + a second sum (dirty lines from zero_ certainly written back)
  r      : sum only of a buffer written once at start-up
  rw_idle: zero_ + sum, then a 50 us spin kernel (lets any write-back drain)
  warm   : nothing (inputs L2-resident)."""
import json, statistics, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P

k = int(sys.argv[1]) if len(sys.argv) > 1 else 22
n = 1 << k
plan = P.Plan(W.random(n, 42))
da = torch.from_numpy(W.make_data(n).view(np.int32)).cuda(); db = torch.empty_like(da)
flush = torch.zeros(64 << 20, dtype=torch.int32, device='cuda')
ms = {'rw': lambda: (flush.zero_(), flush.sum()),
      'rw_r': lambda: (flush.zero_(), flush.sum(), flush.sum()),
      'r': lambda: flush.sum(),
      'rw_idle': lambda: (flush.zero_(), flush.sum(), torch.cuda._sleep(100000)),
      'warm': lambda: None}
for name, pre in ms.items():
    ts = []
    for i in range(45):
        pre()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        if name == 'warm': plan.apply(da, db)
        e0.record(); plan.apply(da, db); e1.record(); torch.cuda.synchronize()
        if i >= 5: ts.append(e0.elapsed_time(e1) * 1e3)
    plan.set_tracing(True)
    w0 = []
    for _ in range(5):
        pre(); plan.apply(da, db); torch.cuda.synchronize()
        tr = plan.trace().astype(np.int64)
        t0 = tr[0][:, 0][tr[0][:, 0] > 0].min()
        w0.append(float(np.median(tr[0][:, 2] - t0)) / 1e3)
        end = max(tr[f][:, 13].max() for f in range(tr.shape[0]))
    plan.set_tracing(False)
    print(json.dumps({'pre': name, 'apply_us': round(statistics.mean(ts), 2),
                      'pass1_first_tile_us_med': round(statistics.median(w0), 2),
                      'span_us': round((end - t0) / 1e3, 2)}), flush=True)
