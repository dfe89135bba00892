# GEMM tile-variant sweep (FEKF_GEMM_VAR bit 0: 128x80 tiles with 16 warps; bit 1: 128x64 / 16 warps for the
# generic path): parity subset, CUPTI kernel table and the bench line per variant
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
for v in 0 1 2 3; do
  FEKF_GEMM_VAR=$v timeout 600 python -m pytest tests/test_parity_gpu.py -q -m gpu -x -k "jacobian or forward or train_steps or graph" -p no:cacheprovider 2>&1 | tail -1 > gpurun_out/gv_test_$v.txt
  FEKF_GEMM_VAR=$v timeout 300 python tools/prof_step.py > gpurun_out/gv_prof_$v.txt 2>/dev/null
  FEKF_GEMM_VAR=$v timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/gv_bench_$v.json 2>/dev/null
done
for v in 0 1 2 3; do echo "== var $v"; cat gpurun_out/gv_test_$v.txt; python tools/bench_brief.py gpurun_out/gv_bench_$v.json; grep "dgemm\|wall\|splitk\|act_bwd\|colsum\|tscan\|tcount" gpurun_out/gv_prof_$v.txt | head -16; done
