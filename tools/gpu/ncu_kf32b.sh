python -m paper_conf_ppopp_huzslmlwtj24_b200.build
N="ncu --kernel-name-base demangled --clock-control none"
timeout 600 $N --set full --import-source on -k regex:kf_pass --launch-skip 4 -c 1 -o gpurun_out/kf32b_ro python tools/kf_bench.py --block 10240 --params 1027082 --precision 32 --defer 15 --iters 4 --warmup 3 > gpurun_out/kf32b.log 2>&1
ls -la gpurun_out/kf32b_ro.ncu-rep
