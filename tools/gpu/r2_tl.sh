# energy-update timeline (fp64), fp32-variant split sweep
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
PROF_UPDATE=0 timeout 300 python tools/prof_step.py > gpurun_out/prof64_u0.txt 2>/dev/null
sed -n '/timeline/,$p' gpurun_out/prof64_u0.txt | awk '$2 > 15' | head -70
for v in 64 80 96 112; do
  FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --precision 32 > gpurun_out/b32_split_$v.json 2>/dev/null
  echo "fp32 split $v: $(python tools/bench_brief.py gpurun_out/b32_split_$v.json | head -2 | tr '\n' ' ')"
done
