#!/bin/bash
mkdir -p gpurun_out
{
timeout 600 python scripts/warm_apply.py 24 '[{"layout": 3}, {"layout": 3, "log2c": 13, "h": [1,4,1]}]'
timeout 600 python scripts/warm_apply.py 25 '[{}, {"passes": 3, "layout": 3}, {"passes": 3, "layout": 3, "fuse": 1}]'
timeout 900 python scripts/warm_apply.py 26 '[{}, {"passes": 3, "layout": 3, "log2c": 14, "h": [1,4,1]}]'
} > gpurun_out/explore_r01g.log 2>&1
