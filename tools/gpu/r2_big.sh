python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 65536 8192 65536 8192; do
  FEKF_GEMM_BIG_ROWS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bbig_$v.json 2>/dev/null
  echo "big_rows $v: $(python tools/bench_brief.py gpurun_out/bbig_$v.json | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bbig_$v.json)"
done
FEKF_GEMM_BIG_ROWS=8192 timeout 300 python tools/prof_step.py > gpurun_out/prof_big.txt 2>/dev/null
grep "dgemm" gpurun_out/prof_big.txt | head -8
FEKF_GEMM_BIG_ROWS=8192 timeout 900 python -m pytest tests/test_parity_gpu.py -q -m gpu -x -k "jacobian or train_steps or forward" -p no:cacheprovider 2>&1 | tail -2
