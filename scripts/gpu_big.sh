#!/bin/bash
# large-n session: SG parity tests, then n = 2^27 / 2^28 plan + apply + sampled parity
#   gpurun -- 'bash scripts/gpu_big.sh TAG "27 28" "random bitrev"'
tag=${1:-big}; ks=${2:-"27 28"}; fams=${3:-"random"}
mkdir -p gpurun_out
{
free -g; nproc
timeout 900 python -m pytest tests -m gpu -x -q -k "schedule_from_global or 5pass or config2" 2>&1 | tail -3
for k in $ks; do for f in $fams; do
  timeout 1200 python scripts/big_n.py --k $k --family $f
done; done
} > gpurun_out/big_$tag.log 2>&1
