#!/bin/bash
tag=${1:-s3}
mkdir -p gpurun_out
{
timeout 600 python -m pytest tests/test_gpu_planner.py -x -q 2>&1 | tail -3
PERM_PLANNER_VERBOSE=1 timeout 900 python scripts/plan_times.py 20,20,20,22,26 random,bitrev 2>&1
PERM_PLANNER_VERBOSE=1 timeout 1500 python scripts/big_n.py --k 30 --family bitrev 2>&1 | grep -v "level"
} > gpurun_out/s3_$tag.log 2>&1
bash scripts/gpu_round.sh r01q
