# per-pair concurrent embedding launches: GPU tests, A/B bench (alternating), timeline
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
for r in 1 2; do for v in 0 1; do
  FEKF_PAIR_STREAMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bps_${v}_$r.json 2>/dev/null
  echo "pair streams $v run $r: $(python tools/bench_brief.py gpurun_out/bps_${v}_$r.json 2>/dev/null | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bps_${v}_$r.json)"
done; done
timeout 300 python tools/prof_step.py > gpurun_out/prof_pairs.txt 2>/dev/null
sed -n '/timeline/,$p' gpurun_out/prof_pairs.txt | awk '$1 < 3300' | head -80
