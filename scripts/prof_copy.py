import sys, torch, statistics
sys.path.insert(0, '.')
import paper_conf_icpp_kasagini13_b200 as P
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
for log2n in (20, 22, 24, 26):
    n = 1 << log2n
    a = torch.zeros(n, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
    ts = []
    for i in range(13):
        flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); P.copy_kernel(a, b); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
    tw = []
    for i in range(13):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); P.copy_kernel(a, b); e1.record(); torch.cuda.synchronize()
        if i >= 3: tw.append(e0.elapsed_time(e1) * 1e3)
    print(f"copy 2^{log2n}: cold {statistics.median(ts):.2f} us ({2*n*4/statistics.median(ts)/1e3:.0f} GB/s)  warm {statistics.median(tw):.2f} us ({2*n*4/statistics.median(tw)/1e3:.0f} GB/s)")
