#!/bin/bash
# C5: size sweep 2^16..2^30, all five families (scheduled passes forced: direct = -1), plan
# build vs apply, conventional kernel, full bit-exact check at every size
tag=${1:-sw}
mkdir -p gpurun_out
{
timeout 1200 python scripts/size_sweep.py --k 16,18,20,21,22,23,24,25,26 --families identity,shuffle,random,bitrev,transpose --configs '[{"direct": -1}]' --check
timeout 1200 python scripts/size_sweep.py --k 27,28 --families identity,shuffle,random,bitrev,transpose --configs '[{"direct": -1}]' --check --reps 5
timeout 1500 python scripts/size_sweep.py --k 29 --families bitrev,transpose,random --configs '[{}]' --check --reps 3
timeout 2400 python scripts/size_sweep.py --k 30 --families bitrev,transpose,random --configs '[{}]' --check --reps 3
} > gpurun_out/sweep_$tag.jsonl 2> gpurun_out/sweep_$tag.err
