#!/bin/bash
mkdir -p gpurun_out
{
echo "== tile_io"; timeout 300 python scripts/micro/tile_io.py
echo "== warm apply"; timeout 300 python scripts/warm_apply.py 20,22
} > gpurun_out/explore_r01e.log 2>&1
