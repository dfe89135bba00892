python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 1500 python -m pytest tests -q -m gpu -x -rf -p no:cacheprovider 2>&1 | tail -4
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bseed.json 2>/dev/null
echo "seed 2-row: $(python tools/bench_brief.py gpurun_out/bseed.json | head -2 | tr '\n' ' ') $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/bseed.json)"
timeout 300 python tools/prof_step.py > gpurun_out/prof_seed.txt 2>/dev/null
grep "desc_bwd_seed\|wall" gpurun_out/prof_seed.txt
sed -n '/timeline/,$p' gpurun_out/prof_seed.txt | grep "desc_bwd_seed"
