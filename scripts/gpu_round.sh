#!/bin/bash
# One GPU session: parity tests, the bench line (both arms), the ncu launch list of the
# same bench command and one --set full capture of the dominant kernel.
#   gpurun --timeout 2400 -- 'bash scripts/gpu_round.sh r01b'
tag=${1:-rXX}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_$tag.log 2>&1
echo "gpu tests exit $?" ; tail -3 gpurun_out/gpu_tests_$tag.log
timeout 600 python bench.py > gpurun_out/bench_$tag.json 2> gpurun_out/bench_$tag.err
echo "bench exit $?"; cat gpurun_out/bench_$tag.json | head -c 600; echo
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$tag.json 2>>gpurun_out/bench_$tag.err
echo "ref exit $?"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file gpurun_out/launches_$tag.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-c3 \
  > gpurun_out/ncu_launch_bench_$tag.log 2>&1
echo "ncu launches exit $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-tlc} -s 6 -c 3 \
  -o gpurun_out/ncu_full_$tag -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-c3 --families random \
  > gpurun_out/ncu_full_$tag.log 2>&1
echo "ncu full exit $?"
