# ncu --set full of one read-write P pass (15 pending corrections, all SMs): kf_bench water-64 sizes, launch 16
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 ncu --kernel-name-base demangled --clock-control none --set full --import-source on -k regex:kf_pass_kernel -s 15 -c 1 -o gpurun_out/kf_rw python tools/kf_bench.py --params 1027082 --defer 15 --iters 16 --warmup 3 > /dev/null 2>&1
python tools/ncu_brief.py gpurun_out/kf_rw.ncu-rep
ncu -i gpurun_out/kf_rw.ncu-rep --page source --csv --print-source sass > gpurun_out/kf_rw_sass.csv 2>/dev/null
python tools/sass_hot.py gpurun_out/kf_rw_sass.csv | head -50
