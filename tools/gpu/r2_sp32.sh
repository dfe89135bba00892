python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 64 72 80 88 96; do
  FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --precision 32 > gpurun_out/sp32_$v.json 2>/dev/null
  echo "fp32 split $v: $(python tools/bench_brief.py gpurun_out/sp32_$v.json | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/sp32_$v.json)"
done
for v in 88 96 104; do
  FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/sp64_$v.json 2>/dev/null
  echo "fp64 split $v: $(python tools/bench_brief.py gpurun_out/sp64_$v.json | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/sp64_$v.json)"
done
