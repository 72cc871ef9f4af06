import ctypes, os, subprocess, statistics, torch
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, 'bw.so')
subprocess.check_call(['nvcc', '-gencode', 'arch=compute_100a,code=sm_100a', '-O3', '-shared', '-Xcompiler', '-fPIC', '-o', so, os.path.join(here, 'bw.cu')])
lib = ctypes.CDLL(so)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
sink = torch.zeros(1, dtype=torch.int32, device='cuda')
for mb in (16, 32, 64, 256):
    n = mb << 18   # int32 count
    a = torch.ones(n, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
    nv = n // 4
    for kind, name in ((0, 'write'), (2, 'read'), (1, 'copy')):
        for warm in (False, True):
            res = []
            for grid, block in ((148 * 4, 512), (148 * 8, 256)):
                ts = torch.zeros(2 * grid, dtype=torch.int64, device='cuda')
                spans = []
                for it in range(6):
                    if not warm:
                        flush.zero_(); flush.sum()
                    else:
                        if kind == 0: b.zero_()
                        else: a.sum()
                    lib.run(kind, ctypes.c_void_p(a.data_ptr()), ctypes.c_void_p(b.data_ptr()), nv,
                            ctypes.c_void_p(ts.data_ptr()), ctypes.c_void_p(sink.data_ptr()), grid, block)
                    torch.cuda.synchronize()
                    t = ts.cpu().numpy().reshape(-1, 2)
                    if it >= 2: spans.append((t[:, 1].max() - t[:, 0].min()) / 1e3)
                us = statistics.median(spans)
                moved = n * 4 * (2 if kind == 1 else 1)
                res.append(f"{us:6.2f}us {moved / us / 1e3:6.0f}GB/s")
            print(f"{mb:4d} MiB {name:5s} {'warm' if warm else 'cold'}: " + " | ".join(res), flush=True)
