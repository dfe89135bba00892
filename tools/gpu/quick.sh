# quick iteration: build, gpu parity tests, bench line (+ optional extra command in $EXTRA)
set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.log 2>&1
if [ -n "$EXTRA" ]; then bash -c "$EXTRA"; fi
cat gpurun_out/pytest_gpu.log; grep '^{' gpurun_out/bench.log | cut -c1-300
