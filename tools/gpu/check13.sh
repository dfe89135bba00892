python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider -x 2>&1 | grep -E "^FAILED|^E  |passed|failed" | head -20
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_fp64.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
grep -h '^{' gpurun_out/bench_fp64.log | cut -c1-200
