python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
for r in 1 2; do for v in 0 1; do
  FEKF_PAIR_STREAMS_W=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bpw_${v}_$r.json 2>/dev/null
  echo "pair streams W $v run $r: $(python tools/bench_brief.py gpurun_out/bpw_${v}_$r.json | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bpw_${v}_$r.json)"
done; done
for v in 100 104; do
  FEKF_SPLIT_SMS=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bpw_s$v.json 2>/dev/null
  echo "pair streams W 1 split $v: $(python tools/bench_brief.py gpurun_out/bpw_s$v.json | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bpw_s$v.json)"
done
