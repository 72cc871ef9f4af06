#!/bin/bash
mkdir -p gpurun_out
{
timeout 900 python scripts/warm_apply.py 22 '[{}, {"h": [2,4,2]}, {"h": [8,8,8]}, {"h": [4,4,4], "stages": 2}, {"h": [2,8,2]}, {"log2c": 10, "h": [8,4,8]}, {"log2c": 12, "h": [2,8,2]}]'
timeout 900 python scripts/warm_apply.py 25 '[{"passes": 3, "layout": 3, "h": [2,4,2]}]'
timeout 900 python scripts/warm_apply.py 20 '[{}, {"h": [8,8,8]}, {"h": [4,4,4]}, {"fuse": 1, "h": [4,4,4]}]'
} > gpurun_out/explore_r01i.log 2>&1
