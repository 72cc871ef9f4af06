#!/bin/bash
tag=${1:-s8}
mkdir -p gpurun_out
{
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 600 python scripts/trace.py --log2n 26 --cfg '{"passes": 5, "log2c": 15}'
timeout 600 python scripts/trace.py --log2n 24 --cfg '{"passes": 5, "log2c": 14}'
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
} > gpurun_out/s8_$tag.log 2>&1
