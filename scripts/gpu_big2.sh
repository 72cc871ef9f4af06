#!/bin/bash
# n = 2^29 / 2^30 (BASELINE configs[3] size, single GPU): plan + apply + sampled parity
tag=${1:-big2}
mkdir -p gpurun_out
{
timeout 900 python scripts/big_n.py --k 29 --family random
timeout 1500 python scripts/big_n.py --k 30 --family bitrev
timeout 1500 python scripts/big_n.py --k 30 --family random
} > gpurun_out/big_$tag.log 2>&1
