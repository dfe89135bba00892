timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_parity_gpu_r2.py -q -m gpu -x -k "kalman or train_steps" -p no:cacheprovider 2>&1 | tail -3
for v in a b; do
  PROF_UPDATE=0 timeout 300 python tools/prof_step.py > gpurun_out/rw2_prof_$v.txt 2>/dev/null
  echo "== $v"; grep "kf_pass" gpurun_out/rw2_prof_$v.txt | head -3
  timeout 300 python tools/kf_bench.py --params 1027082 --defer 15 --iters 16 --warmup 3 > gpurun_out/rw2_kf_$v.json 2>/dev/null; cut -c1-300 gpurun_out/rw2_kf_$v.json
  cp paper_conf_ppopp_huzslmlwtj24_b200/libfekf_cs2.so paper_conf_ppopp_huzslmlwtj24_b200/libfekf.so
done
