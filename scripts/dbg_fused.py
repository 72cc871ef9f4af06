import sys, numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
for k in (18, 20, 22):
    n = 1 << k
    p = W.random(n, k); a = W.make_data(n); ref = scatter_np(p, a)
    for cfg in ({'layout': 2, 'h': (8, 8, 8), 'stages': 2, 'fuse': 1}, {'fuse': -1}, {}, {'layout': 3, 'stages': 1}, {'layout': 3, 'stages': 1, 'fuse': -1}):
        pl = P.Plan(p, **cfg)
        d = pl.describe()
        da = torch.from_numpy(a.view(np.int32)).cuda(); db = torch.full_like(da, -1)
        for rep in range(3):
            db.fill_(-1)
            pl.apply(da, db); torch.cuda.synchronize()
            b = db.cpu().numpy().view(np.uint32)
            bad = np.nonzero(b != ref)[0]
            print(k, cfg, 'fused3', d['fused3'], 'rep', rep, 'mismatches', bad.size, bad[:8], flush=True)
        pl.close()
