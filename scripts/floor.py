"""Where does a 16 MB pass spend its time? copy kernel under different conditions."""
import sys, torch, statistics
sys.path.insert(0, '.')
import paper_conf_icpp_kasagini13_b200 as P
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
tiny = torch.empty(1024, dtype=torch.int32, device='cuda')
def ev(): return torch.cuda.Event(enable_timing=True)
for log2n in (20, 22, 24):
    n = 1 << log2n
    a = torch.zeros(n, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
    res = {}
    for mode in ('cold1', 'cold_after_tiny', 'warm1_busy', 'warm20'):
        ts = []
        for i in range(13):
            if mode == 'cold1':
                flush.zero_(); flush.sum()
            elif mode == 'cold_after_tiny':
                flush.zero_(); flush.sum(); tiny.zero_()
            elif mode == 'warm1_busy':
                flush[: 1 << 20].zero_(); flush[: 8 << 20].sum()   # keep the GPU busy, little eviction
            e0, e1 = ev(), ev()
            e0.record()
            reps = 20 if mode == 'warm20' else 1
            for _ in range(reps):
                P.copy_kernel(a, b)
            e1.record(); torch.cuda.synchronize()
            if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3 / reps)
        res[mode] = statistics.median(ts)
    print(f"copy 2^{log2n} ({2*n*4>>20} MiB moved): " + "  ".join(f"{k}={v:.2f}us" for k, v in res.items()), flush=True)
# empty-ish kernel: copy of 1024 elements
a = torch.zeros(1024, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
ts = []
for i in range(23):
    flush[: 1 << 20].zero_()
    e0, e1 = ev(), ev(); e0.record(); P.copy_kernel(a, b); e1.record(); torch.cuda.synchronize()
    if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
print(f"tiny kernel between events: {statistics.median(ts):.2f} us")
