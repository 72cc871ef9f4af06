#!/bin/bash
mkdir -p gpurun_out
{ echo "== tile_io"; timeout 300 python scripts/micro/tile_io.py; } > gpurun_out/explore_r01f.log 2>&1
