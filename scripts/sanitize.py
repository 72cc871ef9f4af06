"""One small apply through EVERY kernel of libperm, each checked bit-exact with numpy's
b[p] = a: the workload compute-sanitizer runs (memcheck / racecheck / synccheck):

    compute-sanitizer --tool racecheck python scripts/sanitize.py

Kernels covered: fused single-CTA, cluster path, TLC passes (three
launches and the single-launch variant), 5-pass TMA slots (schedule in the slot and
read from global), half-line ring (staged schedule chunks and the re-decoding
variant), plain row pass, 32x32 and 64x64 transposes, TILED layout, sharded steps,
D-/S-designated baselines, block gather, copy.
"""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import workloads as W
import paper_conf_icpp_kasagini13_b200 as P
sys.path.insert(0, 'scripts')
from nphelp import scatter_np, inverse_np

CASES = [
    ("fused_kernel", 12, dict()),
    ("cluster_kernel C=8", 15, dict(passes=2, cluster=8)),
    ("cluster_kernel C=16", 16, dict(passes=2, cluster=16)),
    ("row_pass_tlc_kernel x3", 16, dict(passes=3, layout=3)),
    ("fused_tlc_kernel", 16, dict(passes=3, layout=3, fuse=1)),
    ("row_pass_tma_kernel + transpose64", 16, dict(passes=5)),
    ("row_pass_tma_kernel SG (schedule from global)", 16, dict(passes=5, no_tma=-1, sched_format=2)),
    ("row_pass_split_stg_kernel (staged half-line ring)", 19, dict(passes=5, no_tma=-2, log2c=14, sched_format=0)),
    ("row_pass_split_kernel (re-decoding half-line ring)", 16, dict(passes=5, no_tma=-2, sched_format=-1)),
    ("row_pass_kernel (plain) + transpose", 16, dict(passes=5, no_tma=1)),
    ("row_pass_kernel TILED layout", 16, dict(passes=3, layout=1)),
    ("transpose_kernel 32x32 (view side 32)", 11, dict(passes=5)),
]

only = sys.argv[1] if len(sys.argv) > 1 else ""      # substring filter on the case name
fails = 0
for name, k, kw in CASES:
    if only and only not in name:
        continue
    n = 1 << k
    p = W.random(n, k)
    a = W.make_data(n)
    with P.Plan(p, direct=-1, **kw) as plan:
        da = torch.from_numpy(a.view(np.int32)).cuda()
        db = torch.full_like(da, -1)
        plan.apply(da, db)
        torch.cuda.synchronize()
        ok = np.array_equal(db.cpu().numpy().view(np.uint32), scatter_np(p, a))
    fails += not ok
    print(f"{name:55s} n=2^{k}: {'ok' if ok else 'MISMATCH'}", flush=True)

if only:
    print("ALL OK" if fails == 0 else f"{fails} FAILURES", flush=True)
    sys.exit(1 if fails else 0)
# sharded steps (G = 2 virtual ranks on this device) and the baselines / shortcut kernels
from paper_conf_icpp_kasagini13_b200.sharded import apply_virtual
n, G = 1 << 16, 2
p = W.random(n, 5)
a = W.make_data(n)
for form, kw in (("TLC form", {}), ("per-line 5-pass form", {"passes": 5})):
    plans = [P.Plan(p, world=G, rank=g, **kw) for g in range(G)]
    sh = n // G
    a_sh = [torch.from_numpy(a[g * sh:(g + 1) * sh].view(np.int32).copy()).cuda() for g in range(G)]
    b_sh = [torch.full((sh,), -1, dtype=torch.int32, device="cuda") for _ in range(G)]
    snd = [torch.empty(sh, dtype=torch.int32, device="cuda") for _ in range(G)]
    rcv = [torch.empty(sh, dtype=torch.int32, device="cuda") for _ in range(G)]
    apply_virtual(plans, a_sh, b_sh, snd, rcv)
    torch.cuda.synchronize()
    ok = np.array_equal(np.concatenate([x.cpu().numpy().view(np.uint32) for x in b_sh]), scatter_np(p, a))
    fails += not ok
    print(f"{'sharded steps, ' + form + ' (G=2 virtual ranks)':55s} n=2^16: {'ok' if ok else 'MISMATCH'}", flush=True)
    for pl in plans:
        pl.close()

da = torch.from_numpy(a.view(np.int32)).cuda()
db = torch.empty_like(da)
ref = scatter_np(p, a)
P.scatter_baseline(torch.from_numpy(p).cuda(), da, db)
torch.cuda.synchronize()
ok1 = np.array_equal(db.cpu().numpy().view(np.uint32), ref)
P.gather_baseline(torch.from_numpy(inverse_np(p)).cuda(), da, db)
torch.cuda.synchronize()
ok2 = np.array_equal(db.cpu().numpy().view(np.uint32), ref)
with P.Plan(W.identity(n)) as pl:                          # block gather (direct 3)
    pl.apply(da, db)
    torch.cuda.synchronize()
    ok3 = np.array_equal(db.cpu().numpy().view(np.uint32), a)
P.copy_kernel(da, db)
torch.cuda.synchronize()
ok4 = torch.equal(da, db)
for nm, o in (("scatter_kernel", ok1), ("gather_kernel", ok2), ("block_gather_kernel", ok3), ("copy_kernel", ok4)):
    fails += not o
    print(f"{nm:55s} n=2^16: {'ok' if o else 'MISMATCH'}", flush=True)
print("ALL OK" if fails == 0 else f"{fails} FAILURES", flush=True)
sys.exit(1 if fails else 0)
