#!/bin/bash
# GPU planner + half-line ring session: parity + checker tests, plan-build times host vs
# GPU, large-n applies
tag=${1:-gp}
mkdir -p gpurun_out
{
nproc
timeout 900 python -m pytest tests/test_gpu_planner.py -x -q 2>&1 | tail -15
timeout 900 python -m pytest tests -m gpu -x -q -k "half_line_ring or multi_pass or 5pass or schedule_from_global or config2 or virtual_ranks" 2>&1 | tail -15
timeout 1200 python scripts/plan_times.py 16,18,20,22,24,26 random,bitrev,identity host
timeout 900 python scripts/plan_times.py 28 random
timeout 900 python scripts/big_n.py --k 28 --family random
timeout 1500 python scripts/big_n.py --k 30 --family bitrev
} > gpurun_out/gp_$tag.log 2>&1
