timeout 1200 python -m pytest tests/test_gpu_spos.py tests/test_gpu_spos_kernels.py -q -s -p no:cacheprovider -k "not multistep" > gpurun_out/r2_gputest7.log 2>&1; echo "pytest rc=$?"; grep -E "passed|failed" gpurun_out/r2_gputest7.log | tail -2; grep -E "^FAILED" gpurun_out/r2_gputest7.log | head
# round-2 profiling pass (evidence for profiles/): launch lists of one bench step per
# workload (ncu gpu__time_duration, serialised cold-cache) and ncu --set full captures of
# the dominant kernels inside the timed region (NASPIPE_PROFILE_RANGE=1 + --profile-from-start off).
set -x
ARGS="--steps 2 --warmup 1 --no-cpu --no-secondary --no-repro --no-e2e --no-profile"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches_spos.csv python bench.py $ARGS > /dev/null 2>&1; echo "launch list spos rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches_tf.csv python bench.py --workload transformer $ARGS > /dev/null 2>&1; echo "launch list tf rc=$?"
export NASPIPE_PROFILE_RANGE=1
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"bn_apply_kernel|bn_bwd_apply_kernel|bn_bwd_reduce_kernel|gemm_tc_kernel|dw_tile_kernel|dw_wgrad" -c 40 -o gpurun_out/r2_ncu_spos python bench.py $ARGS > gpurun_out/r2_ncu_spos.log 2>&1; echo "ncu spos rc=$?"
ncu -i gpurun_out/r2_ncu_spos.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,dram__throughput.avg.pct_of_peak_sustained_elapsed,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active > gpurun_out/r2_ncu_spos_raw.csv 2>/dev/null
timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:"gemm_pair_kernel|gemm_tc_kernel|attn_" -c 30 -o gpurun_out/r2_ncu_tf python bench.py --workload transformer $ARGS > gpurun_out/r2_ncu_tf.log 2>&1; echo "ncu tf rc=$?"
ncu -i gpurun_out/r2_ncu_tf.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,dram__throughput.avg.pct_of_peak_sustained_elapsed,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active > gpurun_out/r2_ncu_tf_raw.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep   # > 64 MiB: gpurun would not copy gpurun_out back
ls -la gpurun_out/ | grep r2_
timeout 1200 python bench.py > gpurun_out/r2_bench6.json 2> gpurun_out/r2_bench6.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench6.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches']/d['steps'],d['fractions']); [print(k) for k in d['kernels_top']]; print({k:(v.get('value'),v.get('error'),(v.get('roofline') or {}).get('frac')) for k,v in d['secondary'].items()})"
