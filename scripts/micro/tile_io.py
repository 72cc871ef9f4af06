"""Driver for tile_io.cu: store-pattern costs of a TLC pass skeleton at n = 2^22."""
import ctypes, os, subprocess, statistics, sys
import torch
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, 'tile_io.so')
src = os.path.join(here, 'tile_io.cu')
if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
    subprocess.check_call(['nvcc', '-gencode', 'arch=compute_100a,code=sm_100a', '-O3', '-shared', '-Xcompiler',
                           '-fPIC', '-o', so, src, '-lcuda'])
lib = ctypes.CDLL(so)
n = 1 << 22
inp = torch.arange(n, dtype=torch.int32, device='cuda')
out = torch.empty(n, dtype=torch.int32, device='cuda')
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')
s = torch.cuda.current_stream()

def launch(mode, NA, NB, inflight, grid=148):
    rc = lib.run(ctypes.c_void_p(inp.data_ptr()), ctypes.c_void_p(out.data_ptr()), 512, NA, NB, mode, inflight, grid,
                 ctypes.c_void_p(s.cuda_stream))
    assert rc == 0, rc

def t_cold(fn, reps=10):
    ts = []
    for i in range(reps + 2):
        flush.zero_(); flush.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 2: ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)

def t_warm(fn, k=20):
    fn(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(k): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / k

names = {0: 'bulk1d', 1: 'tensor3d', 2: 'warp-v4', 3: 'no-store', 4: 'reg-direct', 5: 'tensor2d', 6: 'cons-v4'}
# correctness of the X1 geometry (modes 1, 2, 4 must agree)
ref = None
for mode in (1, 2, 4, 5, 6):
    out.zero_(); launch(mode, 4, 2, 1); torch.cuda.synchronize()
    if ref is None: ref = out.clone()
    else: print(f"mode {names[mode]} == tensor3d: {bool(torch.equal(out, ref))}")
print(f"tiny empty-ish floor (mode 3, 1 tile): {t_cold(lambda: lib.run(ctypes.c_void_p(inp.data_ptr()), ctypes.c_void_p(out.data_ptr()), 1, 4, 2, 3, 1, 148, ctypes.c_void_p(s.cuda_stream))):.2f} us")
for mode in (3, 0, 5, 6, 4, 1):
    for NA, NB, infl in ((3, 3, 1), (4, 2, 1), (4, 2, 0), (5, 1, 0), (3, 3, 2), (2, 4, 3)):
        if mode in (3, 4, 6) and (NB != 2 or infl != 1): continue
        if NB == 1 and mode == 2: continue
        f = lambda: launch(mode, NA, NB, infl)
        tc, tw = t_cold(f), t_warm(f)
        print(f"{names[mode]:>10} NA={NA} NB={NB} inflight={infl}: cold {tc:6.2f} us  warm(b2b) {tw:6.2f} us  "
              f"({2*n*4/tw/1e3:6.0f} GB/s warm)", flush=True)
