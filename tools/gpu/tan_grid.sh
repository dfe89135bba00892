python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for g in 0 16 48; do echo "FEKF_TAN_GRID=$g"; FEKF_TAN_GRID=$g python tools/prof_step.py 2>/dev/null | grep -A0 "emb_fwd\|wall per step" | head -3; FEKF_TAN_GRID=$g python tools/prof_step.py 2>/dev/null | sed -n '/timeline/,$p' | grep emb_fwd; done
