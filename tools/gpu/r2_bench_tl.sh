python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python tools/prof_step.py > gpurun_out/prof_step.txt 2>/dev/null
python tools/bench_brief.py gpurun_out/bench.json; head -3 gpurun_out/prof_step.txt; sed -n '/timeline of update 2/,$p' gpurun_out/prof_step.txt | awk '$1>2200 && $2>40'
