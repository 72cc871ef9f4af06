#!/bin/bash
mkdir -p gpurun_out
{
timeout 1200 python -m pytest tests -m gpu -x -q -k "tlc" 2>&1 | tail -3
echo "== trace fuse"; timeout 300 python scripts/trace.py --log2n 22 --cfg '{"fuse": 1}'
echo "== trace fuse 2^20"; timeout 300 python scripts/trace.py --log2n 20 --cfg '{"fuse": 1}'
} > gpurun_out/explore_r01l.log 2>&1
