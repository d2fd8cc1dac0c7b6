#!/bin/bash
# Round-2 (second session) evidence pass: GPU suite, smoke, default bench, launch lists, ncu
# --set full of the dominant kernels inside the bench's timed region, CUPTI kernel tables.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/r2b
O=gpurun_out/r2b
NCU=/usr/local/cuda/bin/ncu
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/gputest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/gputest.log
timeout 1200 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench rc=$?"
ARGS="--steps 2 --warmup 1 --no-cpu --no-secondary --no-repro --no-e2e --no-profile"
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_spos.csv python bench.py $ARGS > /dev/null 2>&1; echo "launch list spos rc=$?"
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_tf.csv python bench.py --workload transformer $ARGS > /dev/null 2>&1; echo "launch list tf rc=$?"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
export NASPIPE_PROFILE_RANGE=1
timeout 900 $NCU --set full --clock-control none --import-source on --profile-from-start off -k regex:"bn_apply_kernel|bn_bwd_apply_kernel|bn_bwd_reduce_kernel" -c 90 -o $O/ncu_spos_bn -f python bench.py $ARGS > $O/ncu_spos_bn.log 2>&1; echo "ncu spos bn rc=$?"
$NCU -i $O/ncu_spos_bn.ncu-rep --page raw --csv --metrics $M > $O/ncu_spos_bn_raw.csv 2>/dev/null
timeout 900 $NCU --set full --clock-control none --import-source on --profile-from-start off -k regex:"gemm_pair_kernel|gemm_tc_kernel|attn_" -c 40 -o $O/ncu_tf -f python bench.py --workload transformer $ARGS > $O/ncu_tf.log 2>&1; echo "ncu tf rc=$?"
$NCU -i $O/ncu_tf.ncu-rep --page raw --csv --metrics $M > $O/ncu_tf_raw.csv 2>/dev/null
unset NASPIPE_PROFILE_RANGE
rm -f $O/*.ncu-rep
timeout 300 python tools/kernel_table.py spos 10 > $O/ktab_spos.txt 2>&1
timeout 300 python tools/kernel_table.py transformer 6 > $O/ktab_tf.txt 2>&1
python -c "import json;d=json.loads(open('$O/bench_default.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches']/d['steps'],d['e2e']['value']); print({k:(v.get('value'),(v.get('roofline') or {}).get('frac')) for k,v in d.get('secondary',{}).items()})"
ls -la $O
