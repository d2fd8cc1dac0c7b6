# ncu --set full of the transformer's small kernels: ln_bwd, sgd_multi, colsum, splitk_reduce, cast_colsum
set -x
mkdir -p gpurun_out
ARGS="--workload transformer --steps 2 --warmup 1 --no-cpu --no-secondary --no-repro --no-e2e --no-profile"
export NASPIPE_PROFILE_RANGE=1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"ln_bwd_kernel|sgd_multi|colsum_bf16|splitk_reduce|cast_colsum|ln_fwd" -c 24 -o gpurun_out/r2_ncu_ln python bench.py $ARGS > gpurun_out/r2_ncu_ln.log 2>&1; echo "ncu rc=$?"
ncu -i gpurun_out/r2_ncu_ln.ncu-rep --page details --csv > gpurun_out/r2_ncu_ln_details.csv 2>/dev/null
ncu -i gpurun_out/r2_ncu_ln.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__average_warp_latency_issue_stalled_long_scoreboard,smsp__pcsamp_warps_issue_stalled_long_scoreboard > gpurun_out/r2_ncu_ln_raw.csv 2>/dev/null
ncu -i gpurun_out/r2_ncu_ln.ncu-rep --page source --csv -k regex:ln_bwd_kernel > gpurun_out/r2_ncu_ln_src.csv 2>/dev/null
rm -f gpurun_out/r2_ncu_ln.ncu-rep
echo done
