# round-2 final artifacts (final: fp32 nets, per-pair streams, fp32 pass products, g_I staging): gpu tests, smoke, bench (fp64, fp32, fp32-P/fp64-nets,
# reference arm), launch list, ncu --set full of the dominant kernels (fp64 and the fp32 nets' GEMM / emb),
# C3/C4 throughput sweep.  Outputs under gpurun_out/r2d/.
set -x
O=gpurun_out/r2d; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > $O/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > $O/pytest_gpu.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/smoke.log 2>&1
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --precision 32 --no-cpu-baseline > $O/bench_fp32.json 2> $O/bench_fp32.err
timeout 600 python bench.py --precision 32 --net-precision 64 --no-cpu-baseline > $O/bench_fp32p.json 2> $O/bench_fp32p.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
$B > /dev/null 2>&1 && timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1500 --csv --log-file $O/launches.csv python bench.py --steps 3 --warmup 0 --no-e2e --no-cpu-baseline > $O/ncu_launch.log 2>&1
N="ncu --kernel-name-base demangled --clock-control none --set full --import-source on"
for k in "kf_pass_kernel 2 kf_pass" "emb_bwd_kernel 7 emb_bwd" "emb_fwd_kernel 3 emb_fwd" "dgemm 0 dgemm_fwd" "desc_bwd_seed_kernel 1 desc_seed_dual"; do
  set -- $k
  timeout 900 $N -k regex:$1 -s $2 -c 1 -o $O/$3 $B > /dev/null 2>&1
  python tools/ncu_brief.py $O/$3.ncu-rep > $O/ncu_$3.txt 2>&1
done
B32="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --precision 32"
$B32 > /dev/null 2>&1
for k in "kf_pass_kernel 2 kf_pass_fp32" "emb_bwd_kernel 7 emb_bwd_fp32" "sgemm_kernel 0 sgemm_fwd_fp32"; do
  set -- $k
  timeout 900 $N -k regex:$1 -s $2 -c 1 -o $O/$3 $B32 > /dev/null 2>&1
  python tools/ncu_brief.py $O/$3.ncu-rep > $O/ncu_$3.txt 2>&1
done
: > $O/c4_bench.jsonl
for c in c4_al32 c4_si72 c4_nacl64 c4_mg36 c4_h2o48 c4_alloy108 c3a_cu108 c3b_ch4; do
  timeout 600 python bench.py --config $c --no-cpu-baseline >> $O/c4_bench.jsonl 2> $O/bench_$c.err
done
tail -3 $O/pytest_gpu.log; cat $O/smoke.log; for f in bench bench_fp32 bench_fp32p; do python tools/bench_brief.py $O/$f.json; done; cut -c1-300 $O/bench_ref.json
timeout 1200 python tools/kf_bench.py --sweep > $O/kf_sweep.jsonl 2> $O/kf_sweep.err
timeout 600 python tools/time_to_rmse.py --config c1_cu32 --max-steps 300 --every 20 --full > $O/ttr_c1.json 2> $O/ttr_c1.err
tail -3 $O/kf_sweep.jsonl; tail -c 300 $O/ttr_c1.json
