python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 ncu --kernel-name-base demangled --clock-control none --set full --import-source on -k regex:desc_fwd_kernel -s 1 -c 2 -o gpurun_out/dfwd python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_brief.py gpurun_out/dfwd.ncu-rep
ncu -i gpurun_out/dfwd.ncu-rep --page source --csv --print-source sass > gpurun_out/dfwd_sass.csv 2>/dev/null
python tools/sass_hot.py gpurun_out/dfwd_sass.csv 0 | head -40
python tools/sass_hot.py gpurun_out/dfwd_sass.csv 1 | head -40
