#!/bin/bash
tag=${1:-s6}
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests -m gpu -x -q -k "staged_schedule or half_line_ring or tall_views" 2>&1 | tail -3
timeout 1800 python scripts/split_variants.py 30 bitrev s512,r512
timeout 900 env PERM_SPLIT=s512 python scripts/big_n.py --k 29 --family random
} > gpurun_out/s6_$tag.log 2>&1
