python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for d in 7 9 11 13 15 11; do
  timeout 300 python bench.py --steps 16 --warmup 3 --no-e2e --no-cpu-baseline --precision 32 --p-defer $d > gpurun_out/bd32_$d.json 2>/dev/null
  echo "fp32 p_defer $d: $(python tools/bench_brief.py gpurun_out/bd32_$d.json | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bd32_$d.json)"
done
for d in 11 13 15 11 15; do
  timeout 300 python bench.py --steps 16 --warmup 3 --no-e2e --no-cpu-baseline --p-defer $d > gpurun_out/bd64_$d.json 2>/dev/null
  echo "fp64 p_defer $d: $(python tools/bench_brief.py gpurun_out/bd64_$d.json | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bd64_$d.json)"
done
