python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 80 88 96 104 112 120; do
  FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_split_$v.json 2>/dev/null
  echo "split $v: $(python tools/bench_brief.py gpurun_out/bench_split_$v.json | head -2 | tr '\n' ' ')"
done
