python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 0 4 8 16; do
  FEKF_L2PF=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_pf_$v.json 2>/dev/null
  echo "pf $v: $(python tools/bench_brief.py gpurun_out/bench_pf_$v.json 2>/dev/null | head -2 | tr '\n' ' ')"
done
