# ncu --set full of the SPOS BN apply kernels (one bench step)
set -x
ARGS="--steps 2 --warmup 1 --no-cpu --no-secondary --no-repro --no-e2e --no-profile"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"bn_apply_kernel|bn_bwd_apply_kernel|bn_bwd_reduce" -s 200 -c 6 -o gpurun_out/r2_ncu_bn python bench.py $ARGS > gpurun_out/r2_ncu_bn.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/r2_ncu_bn.log
ncu -i gpurun_out/r2_ncu_bn.ncu-rep --page details --csv > gpurun_out/r2_ncu_bn_details.csv 2>/dev/null; echo done
