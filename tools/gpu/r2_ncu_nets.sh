# nets kernels: launch list of one bench step + ncu --set full on the new emb_fwd and the 128x80 fitting GEMM
nvidia-smi --query-gpu=memory.used,memory.total --format=csv
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1300 --csv --log-file gpurun_out/launches_nets.csv $B > gpurun_out/ncu_list.log 2>&1
N="ncu --kernel-name-base demangled --clock-control none --set full --import-source on"
timeout 600 $N -k regex:emb_fwd_kernel -s 4 -c 2 -o gpurun_out/emb_fwd2 $B > gpurun_out/ncu_fwd.log 2>&1
timeout 600 $N -k regex:dgemm_kernel -s 0 -c 3 -o gpurun_out/dgemm2 $B > gpurun_out/ncu_gemm.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x -rf 2>&1 | tail -15 > gpurun_out/pytest_all.log
cat gpurun_out/pytest_all.log
nvidia-smi --query-gpu=memory.used,memory.total --format=csv
