# fp32 nets (reading Z22): microbench of the fp32 primitives, fp32 parity tests, full GPU suite, bench lines
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/fp32_peak.cu -o /tmp/fp32_peak && /tmp/fp32_peak > gpurun_out/fp32_peak.json
cat gpurun_out/fp32_peak.json
timeout 900 python -m pytest tests/test_parity_gpu_fp32.py -q -m gpu -rf -p no:cacheprovider 2>&1 | tail -25 > gpurun_out/pytest_fp32.log
cat gpurun_out/pytest_fp32.log
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider --deselect tests/test_parity_gpu_fp32.py 2>&1 | tail -8 > gpurun_out/pytest_all.log
cat gpurun_out/pytest_all.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench64.json 2> gpurun_out/bench64.err
timeout 600 python bench.py --no-cpu-baseline --precision 32 > gpurun_out/bench32.json 2> gpurun_out/bench32.err
timeout 600 python bench.py --no-cpu-baseline --precision 32 --net-precision 64 > gpurun_out/bench32p.json 2> gpurun_out/bench32p.err
for f in bench64 bench32 bench32p; do python tools/bench_brief.py gpurun_out/$f.json; tail -3 gpurun_out/$f.err; done
