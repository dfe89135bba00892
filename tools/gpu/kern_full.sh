# kern_full.sh REGEX SKIP NAME: ncu --set full of one launch of the matching kernel in one bench step
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 900 ncu --kernel-name-base demangled --clock-control none --set full --import-source on -k regex:$1 -s $2 -c 1 -o gpurun_out/$3 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_brief.py gpurun_out/$3.ncu-rep
