set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu -k "kalman or train_steps" 2>&1 | tail -30 > gpurun_out/pytest_fp32.log
timeout 600 python bench.py --precision 32 --no-cpu-baseline --no-e2e > gpurun_out/bench_fp32.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_fp64.log 2>&1
timeout 900 python tools/kf_bench.py --sweep > gpurun_out/kf_sweep.jsonl 2> gpurun_out/kf_sweep.err
N="ncu --kernel-name-base demangled --clock-control none"
timeout 600 $N --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:kf_pass --launch-skip 1 -c 1 --csv --log-file gpurun_out/kf_rw_traffic.csv python bench.py --p-defer 1 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 $N --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:kf_pass --launch-skip 1 -c 2 --csv --log-file gpurun_out/kf_fp32_traffic.csv python bench.py --precision 32 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 $N --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:kf_pass --launch-skip 1 -c 1 --csv --log-file gpurun_out/kf_fp32_rw_traffic.csv python bench.py --precision 32 --p-defer 1 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
cat gpurun_out/pytest_fp32.log gpurun_out/bench_fp32.log gpurun_out/bench_fp64.log
