set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1
# RW vs RO pass timing in the microbench (defer 1 = every pass RW; defer 5 = 1 RW per 5)
timeout 300 python tools/kf_bench.py --nblocks 20 --defer 1 > gpurun_out/kfb_d1.log 2>&1
timeout 300 python tools/kf_bench.py --nblocks 20 --defer 5 --iters 12 > gpurun_out/kfb_d5.log 2>&1
N="ncu --kernel-name-base demangled --clock-control none"
timeout 600 $N --set full --import-source on -k regex:kf_pass --launch-skip 5 -c 1 -o gpurun_out/kf_rw python tools/kf_bench.py --nblocks 4 --defer 5 --iters 3 > gpurun_out/kf_rw.log 2>&1
timeout 600 $N --set full --import-source on -k regex:emb_fwd --launch-skip 8 -c 1 -o gpurun_out/emb_fwd python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/emb_fwd.log 2>&1
timeout 600 $N --set full --import-source on -k "regex:dgemm_kernel<\(int\)32, \(int\)64, \(int\)8, \(int\)32, \(bool\)0, \(bool\)0" --launch-skip 6 -c 1 -o gpurun_out/fit_fwd python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/fit_fwd.log 2>&1
timeout 600 $N --set full --import-source on -k "regex:dgemm_kernel<\(int\)64, \(int\)64, \(int\)32, \(int\)16, \(bool\)1" --launch-skip 6 -c 1 -o gpurun_out/wgrad python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/wgrad.log 2>&1
cat gpurun_out/pytest_gpu.log gpurun_out/bench.log gpurun_out/kfb_d1.log gpurun_out/kfb_d5.log
