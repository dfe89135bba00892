# ncu captures of the top kernels of the water-64 bench step (run from the repo root on the GPU box)
set -x
python -m paper_conf_ppopp_huzslmlwtj24_b200.build
B="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
N="ncu --kernel-name-base demangled --clock-control none"
timeout 600 $N --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:kf_pass -c 5 --csv --log-file gpurun_out/kf_pass_traffic.csv $B > /dev/null 2>&1
i=0
for k in "dgemm_kernel<64, 64, 32, 16, true, false, fekf::EpiPartial>" "dgemm_kernel<128, 64, 32, 32, false, false, fekf::EpiFwd>" "dgemm_kernel<32, 64, 8, 32, false, false, fekf::EpiFwd>" "dgemm_kernel<64, 64, 32, 16, false, true, fekf::EpiDgradAct>" "emb_seed_atom_kernel" "desc_bwd_kernel"; do
  i=$((i+1))
  timeout 600 $N --set full --import-source on -k "regex:${k//[<>]/.}" --launch-skip 6 -c 1 -o gpurun_out/top$i $B > gpurun_out/top$i.log 2>&1
done
ls -la gpurun_out
