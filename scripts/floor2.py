import sys, torch, statistics
sys.path.insert(0, '.')
import paper_conf_icpp_kasagini13_b200 as P
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
def ev(): return torch.cuda.Event(enable_timing=True)
def bench(fn, busy=True, reps=13):
    ts = []
    for i in range(reps):
        if busy: flush.zero_(); flush.sum()
        e0, e1 = ev(), ev(); e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)
t = torch.zeros(1024, dtype=torch.int32, device='cuda'); t2 = torch.empty_like(t)
print("torch tiny op:", bench(lambda: t2.copy_(t)))
print("libperm tiny copy:", bench(lambda: P.copy_kernel(t, t2)))
print("2x libperm tiny copy:", bench(lambda: (P.copy_kernel(t, t2), P.copy_kernel(t, t2))))
for log2n in (20, 22):
    n = 1 << log2n
    a = torch.zeros(n, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
    print(f"2^{log2n}: torch copy {bench(lambda: b.copy_(a)):.2f}  libperm copy {bench(lambda: P.copy_kernel(a, b)):.2f}  "
          f"2x libperm {bench(lambda: (P.copy_kernel(a, b), P.copy_kernel(b, a))):.2f}")
    # graph of 10 copies
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    P.copy_kernel(a, b); torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        for _ in range(10): P.copy_kernel(a, b, stream=s)
    print(f"2^{log2n}: graph of 10 libperm copies per copy (warm): {bench(lambda: g.replay(), busy=False) / 10:.2f}")
    g2 = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g2, stream=s):
        P.copy_kernel(a, b, stream=s)
    print(f"2^{log2n}: graph of 1 copy, cold: {bench(lambda: g2.replay()):.2f}")
