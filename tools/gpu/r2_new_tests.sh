python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1200 python -m pytest tests/test_parity_gpu.py tests/test_parity_gpu_r2.py -q -m gpu -k "c4_time or wide_fitting" -p no:cacheprovider -rA 2>&1 | grep -E "PASS|FAIL|Error|passed|failed" | head -20
bash tools/gpu/r2_c4ttr.sh c4s_mg36 c4s_si72 c4s_al32
python - <<'PY'
import json
for l in open('gpurun_out/c4_ttr.jsonl'):
    d = json.loads(l)
    print(d['config'], d['reached'], round(d['ms_per_step'], 3), d['oracle_minutes_to_target'], [(s, '%.0e' % x) for s, x in d['dev_vs_oracle']][:8])
PY
