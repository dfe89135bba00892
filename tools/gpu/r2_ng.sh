# fp64 pass with two consumer groups (FEKF_FP64_NG=2) against the default, several early-SM counts
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for cfg in "1 96" "2 80" "2 88" "2 96" "1 96"; do
  set -- $cfg
  FEKF_FP64_NG=$1 FEKF_SPLIT_SMS=$2 timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bng_$1_$2.json 2>/dev/null
  echo "NG $1 split $2: $(python tools/bench_brief.py gpurun_out/bng_$1_$2.json | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bng_$1_$2.json)"
done
