set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -30 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
N="ncu --kernel-name-base demangled --clock-control none"
timeout 600 $N --set full --import-source on -k regex:dgemm --launch-skip 0 -c 1 -o gpurun_out/gemm_fwd0 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/gemm.log 2>&1
cat gpurun_out/pytest_gpu.log gpurun_out/bench.log
