#!/bin/bash
tag=${1:-s9}
mkdir -p gpurun_out
{
timeout 1200 python -m pytest tests -m gpu -x -q -k "staged_schedule or half_line_ring or tall_views or schedule_from_global or virtual_ranks or dense" 2>&1 | tail -3
timeout 600 python scripts/trace.py --log2n 26 --cfg '{"passes": 5, "log2c": 15}' | head -2
timeout 1500 python scripts/big_n.py --k 30 --family bitrev
timeout 900 python scripts/big_n.py --k 29 --family random
} > gpurun_out/s9_$tag.log 2>&1
