"""Apply time at n = 2^k: cold (L2 flushed) vs warm back-to-back (everything L2-resident)."""
import sys, statistics, json
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
import paper_conf_icpp_kasagini13_b200 as P
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
for k in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "22").split(",")]:
    n = 1 << k
    p = W.make_perm("random", n)
    a_host = W.make_data(n)
    ref = scatter_np(p, a_host)
    cfgs = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [{}, {"fuse": 1}]
    for cfg in cfgs:
        kw = dict(cfg)
        if "h" in kw: kw["h"] = tuple(kw["h"])
        try:
            pl = P.Plan(p, **kw)
        except Exception as e:
            print(f"2^{k} {json.dumps(cfg)}: plan failed: {e}", flush=True)
            continue
        a = torch.from_numpy(a_host.view(np.int32)).cuda(); b = torch.empty_like(a)
        for _ in range(3): pl.apply(a, b)
        ts = []
        for i in range(12):
            flush.zero_(); flush.sum()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); pl.apply(a, b); e1.record(); torch.cuda.synchronize()
            if i >= 2: ts.append(e0.elapsed_time(e1) * 1e3)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20): pl.apply(a, b)
        e1.record(); torch.cuda.synchronize()
        ok = bool(np.array_equal(b.cpu().numpy().view(np.uint32), ref))
        inf = pl.info()
        print(f"2^{k} {json.dumps(cfg)}: cold {statistics.median(ts):.2f} us  warm b2b {e0.elapsed_time(e1)*1e3/20:.2f} us"
              f"  bitexact={ok} passes={inf['passes']} view={inf['rows']}x{inf['cols']} h={inf['h']}", flush=True)
        pl.close()
