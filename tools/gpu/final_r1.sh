# round-1 artifacts: gpu tests, smoke, bench (both arms, both precisions), launch list, ncu full of the P pass (ro + rw)
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider 2>&1 | tail -3 > gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/bench.log 2>&1
timeout 600 python bench.py --precision 32 --no-cpu-baseline > gpurun_out/bench_fp32.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.log 2>&1
timeout 900 python tools/kf_bench.py --sweep > gpurun_out/kf_sweep.jsonl 2> gpurun_out/kf_sweep.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
N="ncu --kernel-name-base demangled --clock-control none"
timeout 600 $N --set full --import-source on -k regex:kf_pass --launch-skip 1 -c 1 -o gpurun_out/kf_pass_ro python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/kf_full.log 2>&1
timeout 600 $N --set full -k regex:kf_pass --launch-skip 15 -c 1 -o gpurun_out/kf_pass_rw python tools/kf_bench.py --block 10240 --params 1027082 --defer 15 --iters 14 --warmup 3 > gpurun_out/kf_full_rw.log 2>&1
cat gpurun_out/pytest_gpu.log gpurun_out/smoke.log; grep -h '^{' gpurun_out/bench.log gpurun_out/bench_fp32.log gpurun_out/bench_ref.log | cut -c1-200
