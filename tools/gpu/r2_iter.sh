# iteration: build, all GPU tests, emb_fwd launch times, bench line
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 1500 python -m pytest tests -q -m gpu -x -rf 2>&1 | tail -6 > gpurun_out/pytest_all.log
bash tools/gpu/kern.sh ${1:-emb_fwd} ${2:-12} > gpurun_out/kern.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
cat gpurun_out/pytest_all.log gpurun_out/kern.log; python tools/bench_brief.py gpurun_out/bench.json
