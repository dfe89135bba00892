# final-code refresh of the RLEKF bs=1 comparison and the water-64 GPU training trajectory
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 600 python tools/rlekf_bench.py > gpurun_out/rlekf.json 2> gpurun_out/rlekf.err; cat gpurun_out/rlekf.json
timeout 1500 python tools/time_to_rmse.py --config c2_water64 --max-steps 3000 --every 100 --full > gpurun_out/ttr_water64.json 2> gpurun_out/ttr_water64.err
python -c "
import json; d=json.load(open('gpurun_out/ttr_water64.json')); print('train_s', d['train_s'], 'ms/step', d['ms_per_step'], 'final', d['final_rmse']); print([(s, round(e,4), round(f,4)) for s,e,f in d['trajectory']][:12])"
