python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_parity_gpu_r2.py -q -m gpu -x -k "kalman or train or split or naive or sampled or large" -p no:cacheprovider 2>&1 | tail -2
PROF_UPDATE=0 timeout 300 python tools/prof_step.py > gpurun_out/rw_prof.txt 2>/dev/null
grep "kf_pass" gpurun_out/rw_prof.txt | head -3
timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/rw_bench.json 2>/dev/null
timeout 300 python bench.py --no-cpu-baseline --no-e2e --precision 32 > gpurun_out/rw_bench32.json 2>/dev/null
python tools/bench_brief.py gpurun_out/rw_bench.json; python tools/bench_brief.py gpurun_out/rw_bench32.json
