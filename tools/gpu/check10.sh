python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_fp64.log 2>&1
timeout 600 python bench.py --precision 32 --no-cpu-baseline --no-e2e > gpurun_out/bench_fp32.log 2>&1
grep -h '^{' gpurun_out/bench_fp64.log gpurun_out/bench_fp32.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(d['dtype'], d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline']['avg_launch_ms'], d['roofline']['traffic'], d['clocks'], d.get('e2e'))"
