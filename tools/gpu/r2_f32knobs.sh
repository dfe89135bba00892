python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for cfg in "1 15" "0 15" "1 11" "1 15"; do
  set -- $cfg
  FEKF_SPLIT_E=$1 timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --precision 32 --p-defer $2 > gpurun_out/bk_$1_$2.json 2>/dev/null
  echo "fp32 split_e $1 p_defer $2: $(python tools/bench_brief.py gpurun_out/bk_$1_$2.json | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bk_$1_$2.json)"
done
