# Round-end verification on one B200 (run through gpurun from the repo root):
#   bash scripts/gpu_final_r02.sh <tag>
# smoke, bench line, reference arm, ncu launch list of the bench command (per-kernel times +
# DRAM bytes), one ncu --set full capture of the 2^22 TLC passes, the full GPU suite. Outputs land in gpurun_out/ with the tag in their names.
T=${1:-r02}
python -m paper_conf_icpp_kasagini13_b200.build
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$T.log 2>&1; tail -5 gpurun_out/smoke_$T.log
python bench.py > gpurun_out/bench_$T.log 2>&1; tail -c 400 gpurun_out/bench_$T.log
python bench.py --impl reference > gpurun_out/bench_ref_$T.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu_$T.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:row_pass_tlc --launch-skip 3 --launch-count 3 -o gpurun_out/tlc22_$T python scripts/prof_apply.py --log2n 22 --reps 3 > gpurun_out/ncu_full_$T.log 2>&1
# compute-sanitizer: closed on this GPU pool since round 2b (profiles/r02_sanitize_*.log are the last runs)
python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/gputest_$T.log 2>&1; tail -5 gpurun_out/gputest_$T.log
