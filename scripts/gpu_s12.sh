#!/bin/bash
# block-gather shortcut (direct 3): targeted test, smoke, full GPU suite, bench line,
# ncu launch list of the bench restricted to the apply / baseline kernels
tag=${1:-s12}
mkdir -p gpurun_out
{
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k direct_shortcut 2>&1 | tail -3
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
} > gpurun_out/s12_$tag.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --kernel-name regex:"gather|scatter|row_pass_tlc" -c 400 --csv \
  --log-file gpurun_out/launches_$tag.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e \
  > gpurun_out/ncu_bench_$tag.log 2>&1
