python -m paper_conf_icpp_kasagini13_b200.build
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02.log 2>&1; tail -5 gpurun_out/smoke_r02.log
python bench.py > gpurun_out/bench_r02.log 2>&1; tail -c 400 gpurun_out/bench_r02.log
python bench.py --impl reference > gpurun_out/bench_ref_r02.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_r02.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1
for t in memcheck racecheck synccheck; do timeout 900 compute-sanitizer --tool $t --print-limit 10 python scripts/sanitize.py > gpurun_out/sanitize3_$t.log 2>&1; echo "$t rc=$?"; done
python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/gputest_r02_final.log 2>&1; tail -5 gpurun_out/gputest_r02_final.log
