python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/badapt.json 2>/dev/null
python tools/bench_brief.py gpurun_out/badapt.json | head -2
