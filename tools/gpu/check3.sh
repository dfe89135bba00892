set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -30 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_fp64.log 2>&1
timeout 600 python bench.py --precision 32 --no-cpu-baseline --no-e2e > gpurun_out/bench_fp32.log 2>&1
for p in 64 32; do for d in 1 15; do timeout 300 python tools/kf_bench.py --block 10240 --params 1027082 --precision $p --defer $d --iters 16; done; done > gpurun_out/kf_pts.jsonl 2>&1
cat gpurun_out/pytest_gpu.log; grep -h '^{' gpurun_out/bench_fp64.log gpurun_out/bench_fp32.log | cut -c1-400; cat gpurun_out/kf_pts.jsonl | cut -c1-300
