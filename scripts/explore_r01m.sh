#!/bin/bash
mkdir -p gpurun_out
{
timeout 1200 python -m pytest tests -m gpu -x -q -k "tlc" 2>&1 | tail -2
timeout 900 python scripts/warm_apply.py 22,24 '[{}]'
echo "== trace"; timeout 300 python scripts/trace.py --log2n 22
} > gpurun_out/explore_r01m.log 2>&1
