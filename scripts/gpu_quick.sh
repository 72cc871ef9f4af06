#!/bin/bash
# quick GPU iteration: parity tests, per-CTA traces, cold/warm apply times, a short bench
#   gpurun -- 'bash scripts/gpu_quick.sh TAG [pytest -k expr]'
tag=${1:-q}; kexpr=${2:-}
mkdir -p gpurun_out
{
if [ -n "$kexpr" ]; then timeout 900 python -m pytest tests -m gpu -x -q -k "$kexpr" 2>&1 | tail -5;
else timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5; fi
echo "== trace default"; timeout 300 python scripts/trace.py --log2n 22
echo "== trace fuse"; timeout 300 python scripts/trace.py --log2n 22 --cfg '{"fuse": 1}'
echo "== warm apply"; timeout 300 python scripts/warm_apply.py 20,22
timeout 300 python scripts/warm_apply.py 23,24 '[{}, {"layout": 3}, {"layout": 3, "fuse": 1}]'
echo "== bench"; timeout 300 python bench.py --families random,bitrev,transpose --no-cpu-baseline --no-e2e --steps 10
} > gpurun_out/quick_$tag.log 2>&1
