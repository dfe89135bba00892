# iteration: build, all GPU tests, bench line, CUPTI step timeline summary
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 1500 python -m pytest tests -q -m gpu -x -rf 2>&1 | tail -6 > gpurun_out/pytest_all.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python tools/prof_step.py > gpurun_out/prof_step.txt 2>/dev/null
cat gpurun_out/pytest_all.log; python tools/bench_brief.py gpurun_out/bench.json; head -30 gpurun_out/prof_step.txt
