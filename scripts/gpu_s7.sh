#!/bin/bash
tag=${1:-s7}
mkdir -p gpurun_out
{
timeout 1200 python -m pytest tests -m gpu -x -q -k "staged_schedule or half_line_ring or tall_views or gpu_planner or schedule_from_global" 2>&1 | tail -3
PERM_PLANNER_VERBOSE=1 timeout 600 python scripts/plan_times.py 22,26 random 2>&1 | grep -v "level\|\[gplan\] E=\|bank colour\|row colour"
timeout 1500 python scripts/big_n.py --k 30 --family random
} > gpurun_out/s7_$tag.log 2>&1
