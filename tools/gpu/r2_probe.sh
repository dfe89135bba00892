# trajectory divergence probe + nets launch list + C4 throughput
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
timeout 600 python tools/time_to_rmse.py --max-steps 320 --every 8 --full > gpurun_out/ttr_c1.json 2>gpurun_out/ttr_c1.err
for c in c4_al32 c4_si72 c4_nacl64 c4_mg36 c4_h2o48 c4_alloy108 c3a_cu108 c3b_ch4; do
  timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.json 2>gpurun_out/bench_$c.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_r2.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
tail -c 600 gpurun_out/ttr_c1.json; for c in c4_al32 c4_si72 c4_nacl64 c4_mg36 c4_h2o48 c4_alloy108 c3a_cu108 c3b_ch4; do python -c "import json,sys; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value'],1), round(d['ms_per_step'],2), d['roofline_nets'].get('frac'), d['roofline']['frac'])"; done
