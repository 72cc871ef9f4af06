#!/bin/bash
mkdir -p gpurun_out
{
timeout 1500 python scripts/size_sweep.py --k 16,18,20,21,22,23,24,25,26 --families identity,shuffle,random,bitrev,transpose --configs '[{"direct": -1}]' --check
timeout 1500 python scripts/size_sweep.py --k 27,28 --families random,bitrev --configs '[{}]' --reps 5 --check
} > gpurun_out/sweep_r01n.jsonl 2> gpurun_out/sweep_r01n.err
