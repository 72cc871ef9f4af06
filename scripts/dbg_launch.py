import sys, numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np
for k, passes, h in [(12,3,(0,0,0)),(12,5,(0,0,0)),(16,3,(0,0,0)),(16,5,(0,0,0)),(22,3,(0,0,0)),(22,5,(0,0,0))]:
    n = 1 << k
    p = W.bitrev(n); a = W.make_data(n)
    try:
        pl = P.Plan(p, passes=passes, h=h)
        info = pl.info()
        da = torch.from_numpy(a.view(np.int32)).cuda(); db = torch.empty_like(da)
        pl.apply(da, db); torch.cuda.synchronize()
        ok = np.array_equal(db.cpu().numpy().view(np.uint32), scatter_np(p, a))
        print(k, passes, info['h'], 'ok' if ok else 'MISMATCH', flush=True)
    except Exception as e:
        print(k, passes, 'ERR', e, flush=True)
