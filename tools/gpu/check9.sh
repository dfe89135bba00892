python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
FEKF_NG64=2 timeout 900 python -m pytest tests -x -q -m gpu -k "kalman" 2>&1 | tail -3
echo NG1; python tools/gpu/kfexp.py
echo NG2; FEKF_NG64=2 python tools/gpu/kfexp.py
