#!/bin/bash
tag=${1:-s10}
mkdir -p gpurun_out
{
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e
} > gpurun_out/s10_$tag.log 2>&1
