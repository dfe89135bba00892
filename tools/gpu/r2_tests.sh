# Round-2 GPU check: new parity tests first (verbose failures), then the rest, smoke, a quick bench.
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
free -g | head -2; nproc
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 1500 python -m pytest tests/test_parity_gpu_r2.py -q -m gpu -rf --durations=15 2>&1 | tail -60 > gpurun_out/pytest_r2.log
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_bench_gpu.py -q -m gpu -rf --durations=10 2>&1 | tail -40 > gpurun_out/pytest_r1.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1
cat gpurun_out/pytest_r2.log gpurun_out/pytest_r1.log gpurun_out/smoke.log; tail -c 1500 gpurun_out/bench.log
