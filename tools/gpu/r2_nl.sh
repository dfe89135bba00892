python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench64.json 2> gpurun_out/bench64.err
python tools/bench_brief.py gpurun_out/bench64.json
timeout 300 python tools/prof_step.py > gpurun_out/prof64.txt 2>/dev/null
grep "nlist\|wall" gpurun_out/prof64.txt
