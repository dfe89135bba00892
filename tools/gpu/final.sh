# round artifacts: gpu tests, smoke, bench (default), reference arm, ncu launch list of the bench
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/bench.log 2>&1
timeout 600 python bench.py --precision 32 --no-cpu-baseline > gpurun_out/bench_fp32.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1200 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
cat gpurun_out/pytest_gpu.log gpurun_out/smoke.log; grep '^{' gpurun_out/bench.log | cut -c1-400
