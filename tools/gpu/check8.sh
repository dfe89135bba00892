python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu -k "kalman or train_steps or graph" 2>&1 | tail -5
python tools/gpu/kfexp.py
