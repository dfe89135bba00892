# session re-entry check: gpu tests, bench, and ncu of the net kernels (optimisation input)
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.log 2>&1
N="ncu --kernel-name-base demangled --clock-control none"
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 600 $N --set full --import-source on -k regex:emb_bwd_kernel --launch-skip 8 -c 2 -o gpurun_out/emb_bwd $B > gpurun_out/n1.log 2>&1
timeout 600 $N --set full --import-source on -k regex:emb_fwd_kernel --launch-skip 2 -c 1 -o gpurun_out/emb_fwd $B > gpurun_out/n2.log 2>&1
timeout 600 $N --set full --import-source on -k regex:desc_bwd_seed --launch-skip 1 -c 1 -o gpurun_out/desc_seed $B > gpurun_out/n3.log 2>&1
timeout 600 $N --set full --import-source on -k regex:dgemm -c 8 -o gpurun_out/dgemm $B > gpurun_out/n4.log 2>&1
cat gpurun_out/pytest_gpu.log; grep '^{' gpurun_out/bench.log | cut -c1-400
