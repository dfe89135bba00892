# ncu --set full of the fp32 nets' GEMM launches (sgemm_kernel) and the fp64 ones in one bench step
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --precision 32"
N="ncu --kernel-name-base demangled --clock-control none --set full --import-source on"
$B > /dev/null 2>&1 && timeout 900 $N -k regex:sgemm_kernel -s 0 -c 6 -o gpurun_out/sgemm $B > gpurun_out/ncu_sgemm.log 2>&1
python tools/ncu_brief.py gpurun_out/sgemm.ncu-rep
B64="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
$B64 > /dev/null 2>&1 && timeout 900 $N -k regex:dgemm_kernel -s 0 -c 6 -o gpurun_out/dgemm $B64 > gpurun_out/ncu_dgemm.log 2>&1
python tools/ncu_brief.py gpurun_out/dgemm.ncu-rep
