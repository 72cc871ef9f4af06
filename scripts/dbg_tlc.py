"""TLC configurations at small n: bit-exactness per (h, stages, fuse)."""
import sys, json
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
cfgs = json.loads(sys.argv[1])
for c in cfgs:
    k = c.pop("k"); n = 1 << k
    if "h" in c: c["h"] = tuple(c["h"])
    p = W.make_perm(c.pop("fam", "random"), n)
    a = W.make_data(n); ref = scatter_np(p, a)
    try:
        pl = P.Plan(p, passes=3, layout=3, **c)
    except Exception as e:
        print(k, c, "plan failed", e); continue
    da = torch.from_numpy(a.view(np.int32)).cuda(); db = torch.zeros_like(da)
    pl.apply(da, db); torch.cuda.synchronize()
    got = db.cpu().numpy().view(np.uint32)
    bad = np.nonzero(got != ref)[0]
    d = pl.describe()
    print(k, c, "h", pl.info()["h"], "tlc", json.dumps(d.get("tlc")), "mismatches", bad.size, bad[:8], flush=True)
    pl.close()
