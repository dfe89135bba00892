# graph node priorities: split sweep with and without, timeline of a force update with
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for p in 0 1; do for v in 80 96 112; do
  FEKF_GRAPH_PRIO=$p FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bp_${p}_$v.json 2>/dev/null
  echo "prio $p split $v: $(python tools/bench_brief.py gpurun_out/bp_${p}_$v.json | head -2 | tr '\n' ' ')"
done; done
FEKF_GRAPH_PRIO=1 timeout 300 python tools/prof_step.py > gpurun_out/prof_prio.txt 2>/dev/null
sed -n '/timeline/,$p' gpurun_out/prof_prio.txt | awk '$1 > 2400 && $2 > 4' | head -30
for v in 96 112; do
  FEKF_GRAPH_PRIO=1 FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --precision 32 > gpurun_out/bp32_$v.json 2>/dev/null
  echo "fp32 prio split $v: $(python tools/bench_brief.py gpurun_out/bp32_$v.json | head -1)"
done
