#!/bin/bash
# C5 for the low-distribution families with the plan's own choice (auto shortcut: block
# gather for identity, S-designated on P^-1 for shuffle), full bit-exact check at every size
tag=${1:-swd}
mkdir -p gpurun_out
timeout 1200 python scripts/size_sweep.py --k 16,18,20,22,24,26,28 --families identity,shuffle --configs '[{}]' --check --reps 5 \
  > gpurun_out/sweep_$tag.jsonl 2> gpurun_out/sweep_$tag.err
