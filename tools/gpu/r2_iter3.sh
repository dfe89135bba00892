python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf 2>&1 | tail -4
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
python tools/bench_brief.py gpurun_out/bench.json
timeout 300 python tools/kf_bench.py --help > /dev/null 2>&1
PROF_UPDATE=0 timeout 300 python tools/prof_step.py --steps 4 2>/dev/null | grep -m3 "wall\|kf_pass"
