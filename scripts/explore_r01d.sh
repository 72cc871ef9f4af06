#!/bin/bash
mkdir -p gpurun_out
{
echo "== floor2"; timeout 300 python scripts/floor2.py
echo "== floor"; timeout 300 python scripts/floor.py
echo "== trace default"; timeout 300 python scripts/trace.py --log2n 22
echo "== trace fuse"; timeout 300 python scripts/trace.py --log2n 22 --cfg '{"fuse": 1}'
echo "== bench fuse"; timeout 300 python bench.py --families random,bitrev --fuse 1 --no-cpu-baseline --no-e2e --steps 10
} > gpurun_out/explore_r01d.log 2>&1
