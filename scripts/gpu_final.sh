#!/bin/bash
# round-end evidence session: full GPU tests, bench line (+ reference arm, ncu launch list,
# full capture), large-n applies, large-n ncu captures, Table III with 1000 permutations
tag=${1:-r01r}
mkdir -p gpurun_out
bash scripts/gpu_round.sh $tag
{
timeout 900 python scripts/warm_apply.py 22 '[{}, {"stages": 2}, {"stages": 3}, {"fuse": 1}]'
timeout 1200 python scripts/split_variants.py 30 bitrev r512,r1024
timeout 900 python scripts/big_n.py --k 29 --family random
timeout 900 python scripts/big_n.py --k 28 --family bitrev
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
   -k regex:"row_pass|transpose" --csv --log-file gpurun_out/launches_big28_$tag.csv python scripts/big_n.py --k 28 --family random --reps 1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"row_pass_tma|transpose64" -c 2 \
   -o gpurun_out/ncu_big28_$tag -f python scripts/big_n.py --k 28 --family random --reps 1
timeout 1200 python scripts/table3.py --perms 1000 --reps 3
} > gpurun_out/final_$tag.log 2>&1
