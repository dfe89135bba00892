# quick: build, full GPU tests, bench line
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 1500 python -m pytest tests -q -m gpu -x -rf 2>&1 | tail -15 > gpurun_out/pytest_all.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
cat gpurun_out/pytest_all.log; python - <<'PY'
import json
d=json.load(open('gpurun_out/bench.json'))
print("images/s", round(d["value"],1), "ms/step", round(d["ms_per_step"],2), "e2e", d["e2e"] and round(d["e2e"]["value"],1))
print("pass frac", round(d["roofline"]["frac"],3), "alone", round(d["roofline"]["standalone"]["frac"],3), "split", d["roofline"]["split_ms_per_pass"])
n=d["roofline_nets"]; print("nets", {k:(round(v,3) if isinstance(v,float) else v) for k,v in n.items()})
print("clocks", d["clocks"])
PY
