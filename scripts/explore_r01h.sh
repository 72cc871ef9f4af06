#!/bin/bash
mkdir -p gpurun_out
{
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
timeout 600 python scripts/warm_apply.py 22,23,24 '[{}]'
timeout 600 python scripts/warm_apply.py 25 '[{}, {"passes": 3, "layout": 3}]'
timeout 900 python scripts/warm_apply.py 26 '[{"passes": 3, "layout": 3, "log2c": 14, "h": [1,4,1]}]'
} > gpurun_out/explore_r01h.log 2>&1
