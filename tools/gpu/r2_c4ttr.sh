#!/bin/bash
# C4 minutes-to-target on the GPU against the oracle goldens (tests/golden/rmse_c4s_*.json)
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
mkdir -p gpurun_out
: > gpurun_out/c4_ttr.jsonl
for c in "$@"; do
  timeout 600 python tools/time_to_rmse.py --config $c --max-steps 450 --every 20 --full >> gpurun_out/c4_ttr.jsonl 2> gpurun_out/c4_ttr_$c.err
done
