#!/bin/bash
# iteration session: selected GPU tests, plan-build repeat at 2^20, 2^30 apply
tag=${1:-it}
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests/test_gpu_planner.py -x -q 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q -k "half_line_ring or virtual_ranks" 2>&1 | tail -3
timeout 600 python scripts/plan_times.py 20,20,22,20 random,bitrev
timeout 1500 python scripts/big_n.py --k 30 --family bitrev
} > gpurun_out/it_$tag.log 2>&1
