python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 0 1; do
  echo "FEKF_GEMM_6480=$v"
  FEKF_GEMM_6480=$v timeout 300 python tools/prof_step.py 2>/dev/null | grep "wall\|dgemm"
  FEKF_GEMM_6480=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b6480_$v.json 2>/dev/null
  python tools/bench_brief.py gpurun_out/b6480_$v.json | head -1
done
timeout 900 python -m pytest tests/test_parity_gpu.py -q -m gpu -x -k "train_steps or jacobian or forward" 2>&1 | tail -2
FEKF_GEMM_6480=1 timeout 900 python -m pytest tests/test_parity_gpu.py -q -m gpu -x -k "train_steps or jacobian or forward" 2>&1 | tail -2
