# fp32 nets: full GPU suite, per-kernel CUPTI tables fp64 vs fp32 nets, bench lines
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -rf -p no:cacheprovider 2>&1 | tail -8 > gpurun_out/pytest_all.log
cat gpurun_out/pytest_all.log
timeout 300 python tools/prof_step.py > gpurun_out/prof64.txt 2>/dev/null
timeout 300 python tools/prof_step.py --precision 32 > gpurun_out/prof32.txt 2>/dev/null
timeout 300 python tools/prof_step.py --precision 32 --net-precision 64 > gpurun_out/prof32p.txt 2>/dev/null
timeout 600 python bench.py --no-cpu-baseline --precision 32 > gpurun_out/bench32.json 2> gpurun_out/bench32.err
python tools/bench_brief.py gpurun_out/bench32.json
head -30 gpurun_out/prof64.txt; head -30 gpurun_out/prof32.txt
