#!/bin/bash
# large-n kernels: 2^28 / 2^30 applies, ncu launch list + one full capture of the long-line
# row passes and the 64x64 transpose; Table III with 1000 permutations at 4M
tag=${1:-b3}
mkdir -p gpurun_out
{
timeout 600 python -m pytest tests -m gpu -x -q -k "half_line_ring or schedule_from_global" 2>&1 | tail -2
timeout 900 python scripts/big_n.py --k 28 --family random
timeout 1500 python scripts/big_n.py --k 30 --family bitrev
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
   -k regex:"row_pass|transpose" --csv --log-file gpurun_out/launches_big28_$tag.csv python scripts/big_n.py --k 28 --family random --reps 1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"row_pass_tma|transpose64" -c 2 \
   -o gpurun_out/ncu_big28_$tag -f python scripts/big_n.py --k 28 --family random --reps 1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"row_pass_split" -c 1 \
   -o gpurun_out/ncu_big30_$tag -f python scripts/big_n.py --k 30 --family bitrev --reps 1
timeout 1200 python scripts/table3.py --perms 1000 --reps 3
} > gpurun_out/big3_$tag.log 2>&1
