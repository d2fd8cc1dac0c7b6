#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spos_kernels.py -x -q > gpurun_out/s2_kernels.log 2>&1; echo kernels=$?; tail -2 gpurun_out/s2_kernels.log
timeout 300 python tools/kernel_table.py spos 10 > gpurun_out/ktab4_spos.txt 2>&1
timeout 300 python tools/kernel_table.py transformer 6 > gpurun_out/ktab4_tf.txt 2>&1
for i in 1 2; do
timeout 600 python bench.py --steps 40 --warmup 5 --no-secondary --no-cpu --no-repro > gpurun_out/s2_bench_$i.json 2>>gpurun_out/s2_err.log
python -c "import json;d=json.loads(open('gpurun_out/s2_bench_$i.json').read().strip().splitlines()[-1]);print('s2',d['value'],d['ms_per_step'],d['roofline']['frac'],d.get('gpu_launches'))"
done
