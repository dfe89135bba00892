python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider 2>&1 | grep -E "^FAILED|^E  |passed|failed" | head -20
timeout 300 python tools/infer_bench.py --config c2_water64 > gpurun_out/infer_water.log 2>&1
timeout 300 python tools/infer_bench.py --config paper_cu108 > gpurun_out/infer_pcu.log 2>&1
timeout 600 python bench.py --config c3a_cu108 --no-cpu-baseline --no-e2e --steps 5 > gpurun_out/bench_c3a.log 2>&1
timeout 600 python bench.py --config c3b_ch4 --no-cpu-baseline --no-e2e --steps 5 > gpurun_out/bench_c3b.log 2>&1
timeout 600 python bench.py --config paper_cu108 --no-cpu-baseline --no-e2e --steps 10 > gpurun_out/bench_pcu.log 2>&1
cat gpurun_out/infer_water.log gpurun_out/infer_pcu.log; grep -h '^{' gpurun_out/bench_c3a.log gpurun_out/bench_c3b.log gpurun_out/bench_pcu.log | cut -c1-260; tail -3 gpurun_out/bench_c3a.log
