set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -30 > gpurun_out/pytest_gpu.log
for p in 32 64; do for d in 1 15; do timeout 300 python tools/kf_bench.py --block 10240 --params 1027082 --precision $p --defer $d --iters 16; done; done > gpurun_out/kf_pts.jsonl 2>&1
timeout 600 python bench.py --precision 32 --no-cpu-baseline --no-e2e > gpurun_out/bench_fp32.log 2>&1
cat gpurun_out/pytest_gpu.log; cut -c1-330 gpurun_out/kf_pts.jsonl; grep -h '^{' gpurun_out/bench_fp32.log | cut -c1-200
