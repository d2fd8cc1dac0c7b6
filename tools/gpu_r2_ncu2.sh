# ncu details of the transformer's ln_bwd and tcgen05 attention kernels (timed region)
set -x
export NASPIPE_PROFILE_RANGE=1
ARGS="--workload transformer --steps 2 --warmup 1 --no-cpu --no-secondary --no-repro --no-e2e --no-profile"
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"ln_bwd_kernel|attn_bwd_tc|attn_fwd_tc" -c 8 -o gpurun_out/r2_ncu_tf2 python bench.py $ARGS > gpurun_out/r2_ncu_tf2.log 2>&1; echo "ncu rc=$?"
ncu -i gpurun_out/r2_ncu_tf2.ncu-rep --page details --csv > gpurun_out/r2_ncu_tf2_details.csv 2>/dev/null
ncu -i gpurun_out/r2_ncu_tf2.ncu-rep --page source --csv --kernel-name regex:attn_bwd_tc64 --launch-count 1 > gpurun_out/r2_ncu_attn64_source.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
ls -la gpurun_out | grep tf2
