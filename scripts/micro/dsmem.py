"""Driver for dsmem.cu: DSMEM store/load throughput per SM, cluster and grid barrier costs."""
import ctypes, os, subprocess, statistics
import torch
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, 'dsmem.so')
src = os.path.join(here, 'dsmem.cu')
subprocess.check_call(['nvcc', '-gencode', 'arch=compute_100a,code=sm_100a', '-O3', '-shared', '-Xcompiler',
                       '-fPIC', '-o', so, src])
lib = ctypes.CDLL(so)
out = torch.zeros(1024, dtype=torch.int64, device='cuda')
ctr = torch.zeros(1, dtype=torch.int64, device='cuda')
ms = ctypes.c_float()
names = {0: 'local st.u32', 1: 'dsmem st.u32 1 peer/warp', 2: 'dsmem st.u32 lanes->all peers',
         3: 'dsmem ld.u32 1 peer/warp', 4: 'dsmem st.v4 1 peer/warp', 5: 'cluster barrier'}
iters = 200
for csize in (2, 4, 8, 16):
    grid = (148 // csize) * csize if csize <= 8 else 128
    for mode in range(6):
        rc = lib.run_dsmem(mode, csize, grid, iters, ctypes.c_void_p(out.data_ptr()), ctypes.byref(ms))
        if rc != 0:
            print(f"csize {csize} mode {mode}: rc {rc}")
            continue
        cyc = out[:grid].cpu().double()
        med = float(cyc.median())
        if mode == 5:
            print(f"csize {csize:2d} grid {grid}: {names[mode]:32s} {med / iters:8.1f} cyc per barrier", flush=True)
        else:
            byts = 1024 * 64 * iters
            print(f"csize {csize:2d} grid {grid}: {names[mode]:32s} {byts / med:6.1f} B/cyc/SM  "
                  f"aggregate {byts * grid / (ms.value * 1e-3) / 1e12:6.2f} TB/s  ({ms.value * 1e3:.1f} us)", flush=True)
for threads in (64, 576):
    for grid in (148,):
        rc = lib.run_grid_barrier(grid, threads, 1000, ctypes.c_void_p(ctr.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                  ctypes.byref(ms))
        cyc = out[:grid].cpu().double()
        print(f"grid barrier grid {grid} threads {threads}: {float(cyc.median()) / 1000:8.1f} cyc, "
              f"{ms.value * 1e3 / 1000:6.3f} us per barrier (events)", flush=True)
