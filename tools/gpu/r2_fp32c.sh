python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests/test_parity_gpu_fp32.py tests/test_parity_gpu.py -q -m gpu -rf -p no:cacheprovider -k "fp32 or split_pass or train_steps" 2>&1 | tail -6
timeout 300 python tools/prof_step.py --precision 32 > gpurun_out/prof32.txt 2>/dev/null
timeout 600 python bench.py --no-cpu-baseline --precision 32 > gpurun_out/bench32.json 2> gpurun_out/bench32.err
python tools/bench_brief.py gpurun_out/bench32.json
head -24 gpurun_out/prof32.txt
