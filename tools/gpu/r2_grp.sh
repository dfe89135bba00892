python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
for r in 1 2; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bgrp_$r.json 2>/dev/null
  echo "grouped run $r: $(python tools/bench_brief.py gpurun_out/bgrp_$r.json 2>/dev/null | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bgrp_$r.json)"
done
timeout 300 python tools/prof_step.py > gpurun_out/prof_grp.txt 2>/dev/null
head -3 gpurun_out/prof_grp.txt
sed -n '/timeline/,$p' gpurun_out/prof_grp.txt | awk '$1 > 1900 && $1 < 3200'
