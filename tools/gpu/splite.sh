python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 0 1 0 1; do
  FEKF_SPLIT_E=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_se_$v.json 2>/dev/null
  echo "split_e $v: $(python tools/bench_brief.py gpurun_out/bench_se_$v.json 2>/dev/null | head -1)"
done
PROF_UPDATE=0 timeout 300 python tools/prof_step.py 2>/dev/null | sed -n '/timeline of update/,$p' | awk '$2>30'
