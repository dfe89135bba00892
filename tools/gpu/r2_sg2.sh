python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests/test_parity_gpu_fp32.py -q -m gpu -rf -p no:cacheprovider 2>&1 | tail -4
timeout 600 python bench.py --no-cpu-baseline --precision 32 > gpurun_out/bench32.json 2> gpurun_out/bench32.err
python tools/bench_brief.py gpurun_out/bench32.json
timeout 300 python tools/prof_step.py --precision 32 > gpurun_out/prof32.txt 2>/dev/null
grep "wall\|sgemm" gpurun_out/prof32.txt
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --precision 32"
N="ncu --kernel-name-base demangled --clock-control none --set full --import-source on"
$B > /dev/null 2>&1 && timeout 900 $N -k regex:sgemm_kernel -s 0 -c 6 -o gpurun_out/sgemm2 $B > /dev/null 2>&1
python tools/ncu_brief.py gpurun_out/sgemm2.ncu-rep | grep -E "==|time_dur|fma_cyc|issue_active|bank|stalls"
