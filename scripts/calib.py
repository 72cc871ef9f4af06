"""Box calibration: GPU identity, clocks, copy bandwidth (cold/warm) at 2^22 and 2^26."""
import subprocess, sys, statistics, torch
sys.path.insert(0, '.')
import paper_conf_icpp_kasagini13_b200 as P
q = subprocess.run(["nvidia-smi", "--query-gpu=uuid,clocks.sm,clocks.mem,clocks.max.sm,clocks.max.mem,power.draw,temperature.gpu",
                    "--format=csv,noheader"], capture_output=True, text=True).stdout.strip()
print("gpu:", q)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
def ev(): return torch.cuda.Event(enable_timing=True)
for k in (22, 26):
    n = 1 << k
    a = torch.zeros(n, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
    ts = []
    for i in range(13):
        flush.zero_(); flush.sum()
        e0, e1 = ev(), ev(); e0.record(); P.copy_kernel(a, b); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
    e0, e1 = ev(), ev(); e0.record()
    for _ in range(20): P.copy_kernel(a, b)
    e1.record(); torch.cuda.synchronize()
    w = e0.elapsed_time(e1) * 1e3 / 20
    print(f"copy 2^{k}: cold {statistics.median(ts):.2f} us ({2*n*4/statistics.median(ts)/1e3:.0f} GB/s)  warm b2b {w:.2f} us ({2*n*4/w/1e3:.0f} GB/s)")
