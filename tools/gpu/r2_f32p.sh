python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
for p in 64 32; do
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --precision $p > gpurun_out/bf32_$p.json 2>/dev/null
  echo "fp32 products, precision $p: $(python tools/bench_brief.py gpurun_out/bf32_$p.json 2>/dev/null | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bf32_$p.json)"
done
N="ncu --kernel-name-base demangled --clock-control none --set full --import-source on"
B32="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --precision 32"
$B32 > /dev/null 2>&1 && timeout 900 $N -k regex:kf_pass_kernel -s 2 -c 1 -o gpurun_out/kff3232 $B32 > /dev/null 2>&1
python tools/ncu_brief.py gpurun_out/kff3232.ncu-rep | grep -E "==|time_dur|dram__bytes.sum.per|issue_active|stalls"
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 $N -k regex:kf_pass_kernel -s 2 -c 1 -o gpurun_out/kff3264 $B > /dev/null 2>&1
python tools/ncu_brief.py gpurun_out/kff3264.ncu-rep | grep -E "==|time_dur|dram__bytes.sum.per|issue_active|stalls"
