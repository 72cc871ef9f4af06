#!/bin/bash
tag=${1:-s4}
mkdir -p gpurun_out
{
timeout 600 python scripts/ab_planner.py 22 random,bitrev,transpose
timeout 600 python scripts/ab_planner.py 24 random
timeout 600 python scripts/ab_planner.py 26 random
timeout 900 python -m pytest tests -m gpu -x -q -k "half_line_ring or schedule_from_global or virtual_ranks or gpu_planner" 2>&1 | tail -3
timeout 900 python scripts/big_n.py --k 28 --family random
timeout 1500 python scripts/big_n.py --k 30 --family random
} > gpurun_out/s4_$tag.log 2>&1
