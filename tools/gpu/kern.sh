# kern.sh REGEX COUNT [extra bench args]: per-launch time, fp64 pipe, warps of the matching kernels in one bench step
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
M=gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active
timeout 900 ncu --metrics $M --clock-control none -k regex:$1 -c $2 --csv --log-file gpurun_out/kern_$1.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline $3 > /dev/null 2>&1
python tools/kern_table.py gpurun_out/kern_$1.csv
