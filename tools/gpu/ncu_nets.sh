set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
N="ncu --kernel-name-base demangled --clock-control none"
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 $N --set full --import-source on -k regex:emb_bwd_kernel --launch-skip 8 -c 4 -o gpurun_out/emb_bwd $B > gpurun_out/n1.log 2>&1
timeout 600 $N --set full --import-source on -k regex:emb_fwd_kernel -c 1 -o gpurun_out/emb_fwd $B > gpurun_out/n2.log 2>&1
timeout 600 $N --set full --import-source on -k regex:desc_bwd_seed --launch-skip 1 -c 1 -o gpurun_out/desc_seed $B > gpurun_out/n3.log 2>&1
timeout 600 $N --set full -k regex:dgemm -c 6 -o gpurun_out/dgemm $B > gpurun_out/n4.log 2>&1
ls -la gpurun_out/*.ncu-rep
