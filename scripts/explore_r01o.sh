#!/bin/bash
mkdir -p gpurun_out
{
timeout 1200 python -m pytest tests -m gpu -x -q -k "tlc or config1" 2>&1 | tail -2
for v in 0 1; do echo "== LAST_LSU=$v"; PERM_TLC_LAST_LSU=$v timeout 900 python scripts/warm_apply.py 20,22,24 '[{}]'; done
echo "== trace"; timeout 300 python scripts/trace.py --log2n 22
} > gpurun_out/explore_r01o.log 2>&1
