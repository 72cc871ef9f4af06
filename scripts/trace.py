"""Per-CTA phase timeline of one apply (globaltimer stamps), cold L2."""
import argparse, json, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
ap = argparse.ArgumentParser()
ap.add_argument('--log2n', type=int, default=22)
ap.add_argument('--cfg', default='{}')
ap.add_argument('--dump', default='', help='save the raw per-CTA stamps (npz)')
a = ap.parse_args()
n = 1 << a.log2n
p = W.random(n, 42)
kw = json.loads(a.cfg)
if 'h' in kw: kw['h'] = tuple(kw['h'])
plan = P.Plan(p, **kw)
da = torch.from_numpy(W.make_data(n).view(np.int32)).cuda(); db = torch.empty_like(da)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
plan.set_tracing(True)
for _ in range(3):
    flush.zero_(); flush.sum(); plan.apply(da, db)
torch.cuda.synchronize()
tr = plan.trace().astype(np.int64)
if a.dump:
    np.savez(a.dump, trace=tr, describe=json.dumps(plan.describe()))
d = plan.describe()
ts_ = tr[:, :, :15]
t0 = ts_[ts_ > 0].min()          # slot 15 holds the SM id, not a time
names = {0: 'start', 1: 'pdl_ok', 2: 'w0', 3: 'p0', 4: 's0', 5: 'w1', 6: 'p1', 7: 's1', 8: 'w2', 9: 'p2', 10: 's2', 14: 'end'}
print(json.dumps(kw), 'passes', d['passes'], 'layout', d.get('layout'), 'fused3', d.get('fused3'))
if d.get('fused3'):
    t = tr[0]
    t = t[(t[:, 0] > 0)]
    rel = (t - t0) / 1000.0
    fn = {0: 'start'}
    for k in range(3):
        fn.update({1 + 4 * k: f'P{k}data', 2 + 4 * k: f'P{k}perm0', 3 + 4 * k: f'P{k}permEnd', 4 + 4 * k: f'P{k}storeEnd'})
    fn[13] = 'P0proxyFence'; fn[14] = 'P0bulkWait0'
    fn[15] = 'end'
    for c in sorted(fn):
        v = rel[:, c][t[:, c] > 0]
        if v.size:
            print(f"  {fn[c]:>12}: min {v.min():7.2f}  med {np.median(v):7.2f}  max {v.max():7.2f}  (n={v.size})")
    sys.exit(0)
if d.get('layout') == 3:
    names = {0: 'start', 1: 'pdl_ok', 2: 'w0', 4: 's0', 5: 'w1', 7: 's1', 8: 'w2', 10: 's2', 3: 'permEnd', 12: 'sLast',
             13: 'drained', 14: 'end'}
for f in range(3):
    t = tr[f]
    t = t[(t[:, 0] > 0)]
    rel = (t - t0) / 1000.0
    def q(col):
        v = rel[:, col][t[:, col] > 0]
        return f"{v.min():6.2f}/{np.median(v):6.2f}/{v.max():6.2f}" if v.size else "   -   "
    print(f"pass {f}: ctas={t.shape[0]}  " + "  ".join(f"{names[c]}={q(c)}" for c in names))
