"""Event-timed floor of one tiny kernel on this box (what every cold-L2 apply pays on top of
its kernels): a 4 KiB perm_copy_kernel between two CUDA events, after (a) the bench's L2
flush (256 MiB write + read), (b) a write-only flush, (c) no flush; and 1 / 2 / 3 such
launches back to back. Mean of `reps` (the event clock steps in ~1 us quanta here)."""
import json, statistics, sys
import torch
sys.path.insert(0, '.')
import paper_conf_icpp_kasagini13_b200 as P

reps = 200
a = torch.zeros(1024, dtype=torch.int32, device='cuda'); b = torch.empty_like(a)
flush = torch.empty(64 << 20, dtype=torch.int32, device='cuda')


def run(pre, k):
    ts = []
    for i in range(reps + 5):
        pre()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(k): P.copy_kernel(a, b)
        e1.record(); torch.cuda.synchronize()
        if i >= 5: ts.append(e0.elapsed_time(e1) * 1e3)
    return round(statistics.mean(ts), 2)


pres = {'flush_rw': lambda: (flush.zero_(), flush.sum()), 'flush_w': lambda: flush.zero_(),
        'none': lambda: None}
for name, pre in pres.items():
    print(json.dumps({'pre': name, 'us_1': run(pre, 1), 'us_2': run(pre, 2), 'us_3': run(pre, 3)}), flush=True)
