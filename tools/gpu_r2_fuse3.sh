#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spos_kernels.py -x -q > gpurun_out/fuse3_kernels.log 2>&1; echo kernels=$?
tail -3 gpurun_out/fuse3_kernels.log
for cfg in "1 1" "0 0" "1 0" "0 1"; do
  set -- $cfg
  NASPIPE_SPOS_FUSE_BNB=$1 NASPIPE_SPOS_FUSE_BNA=$2 timeout 300 python tools/kernel_table.py spos 10 > gpurun_out/ktab3_$1$2.txt 2>&1
  NASPIPE_SPOS_FUSE_BNB=$1 NASPIPE_SPOS_FUSE_BNA=$2 timeout 600 python bench.py --steps 40 --warmup 5 --no-secondary --no-cpu --no-repro > gpurun_out/fuse3_bench_$1$2.json 2>>gpurun_out/fuse3_err.log
  python -c "import json;d=json.loads(open('gpurun_out/fuse3_bench_$1$2.json').read().strip().splitlines()[-1]);print('bnb=$1 bna=$2',d['value'],d['ms_per_step'],d['roofline']['frac'],d.get('gpu_launches'))"
done
timeout 1500 python -m pytest tests/test_gpu_spos.py tests/test_gpu_policies.py tests/test_gpu_mirror.py tests/test_gpu_multirank.py tests/test_gpu_context.py -x -q > gpurun_out/fuse3_gputest.log 2>&1; echo gputests=$?
tail -3 gpurun_out/fuse3_gputest.log
