import ctypes, os, subprocess, sys, statistics, torch
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, 'store_pattern.so')
if not os.path.exists(so):
    subprocess.check_call(['nvcc', '-gencode', 'arch=compute_100a,code=sm_100a', '-O3', '-shared', '-Xcompiler', '-fPIC', '-o', so, os.path.join(here, 'store_pattern.cu')])
lib = ctypes.CDLL(so)
n = 1 << 22
out = torch.empty(n, dtype=torch.int32, device='cuda')
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
R = 2048; L = 2048
for h in (4, 8, 16, 32):
    for co in (0, 1):
        for grid, block in ((148, 256), (148, 512), (296, 512), (1184, 256)):
            ts = []
            for i in range(8):
                flush.zero_(); flush.sum()
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                e0.record(); lib.run(ctypes.c_void_p(out.data_ptr()), L, R, h, R // h, co, grid, block); e1.record()
                torch.cuda.synchronize()
                if i >= 2: ts.append(e0.elapsed_time(e1) * 1e3)
            t = statistics.median(ts)
            print(f"h={h:2d} {'coalesced' if co else 'column  '} grid={grid:4d} block={block}: {t:6.2f} us  {n*4/t/1e3:7.1f} GB/s", flush=True)
