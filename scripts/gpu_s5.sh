#!/bin/bash
tag=${1:-s5}
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests -m gpu -x -q -k "half_line_ring or schedule_from_global or virtual_ranks" 2>&1 | tail -3
timeout 2400 python scripts/split_variants.py 30 bitrev r1024,k1024,r512,k512
timeout 900 python scripts/big_n.py --k 29 --family random
} > gpurun_out/s5_$tag.log 2>&1
