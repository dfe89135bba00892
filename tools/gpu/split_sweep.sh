# split P pass: gpu tests, then the bench line for several early-pass SM counts (0 = no split)
set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 900 python -m pytest tests -x -q -m gpu -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_gpu.log
for n in ${SPLITS:-0 64 80 96 112 128}; do
  FEKF_SPLIT_SMS=$n timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_split_$n.log 2>&1
  echo "split=$n $(grep '^{' gpurun_out/bench_split_$n.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["roofline"]["frac"])')"
done
cat gpurun_out/pytest_gpu.log
