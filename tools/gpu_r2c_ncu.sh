#!/bin/bash
# ncu evidence on the final code: configs[1] launch list and ncu --set full of the BatchNorm
# family inside the bench's timed region
cd "$(dirname "$0")/.."
O=gpurun_out/r2c_ncu; mkdir -p $O
NCU=/usr/local/cuda/bin/ncu
ARGS="--steps 2 --warmup 1 --no-cpu --no-secondary --no-repro --no-e2e --no-profile"
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_spos.csv python bench.py $ARGS > /dev/null 2>&1; echo "launch list spos rc=$?"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
export NASPIPE_PROFILE_RANGE=1
timeout 1200 $NCU --set full --clock-control none --import-source on --profile-from-start off -k regex:"bn_apply_kernel|bn_bwd_apply_kernel|bn_bwd_reduce_kernel" -c 90 -o $O/ncu_spos_bn -f python bench.py $ARGS > $O/ncu_spos_bn.log 2>&1; echo "ncu spos bn rc=$?"
$NCU -i $O/ncu_spos_bn.ncu-rep --page raw --csv --metrics $M > $O/ncu_spos_bn_raw.csv 2>/dev/null
rm -f $O/*.ncu-rep
ls -la $O
