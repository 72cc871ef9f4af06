#!/bin/bash
mkdir -p gpurun_out
{
python scripts/calib.py; timeout 1200 python -m pytest tests -m gpu -x -q -k "tlc or config1 or every_layout or fused3" 2>&1 | tail -3
timeout 900 python scripts/warm_apply.py 22,23,24,25 '[{}, {"sched_format": -1}]'
echo "== trace default"; timeout 300 python scripts/trace.py --log2n 22
echo "== bench"; timeout 300 python bench.py --families random,bitrev,transpose --no-cpu-baseline --no-e2e --steps 10
} > gpurun_out/explore_r01j.log 2>&1
