#!/bin/bash
# round-2 BatchNorm fusion check: kernel tests, the SPOS/parity suites, A/B bench of the fusion
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spos_kernels.py -x -q > gpurun_out/fuse_kernels.log 2>&1; echo kernels=$?
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/fuse_gputest.log 2>&1; echo gputests=$?
for v in 1 0 1 0; do
  NASPIPE_SPOS_FUSE_BNB=$v timeout 600 python bench.py --steps 40 --warmup 5 --no-secondary --no-cpu --no-repro > gpurun_out/fuse_bench_$v.json 2>>gpurun_out/fuse_bench_err.log
  python -c "import json;d=json.loads(open('gpurun_out/fuse_bench_$v.json').read().strip().splitlines()[-1]);print('fuse=$v',d['value'],d['ms_per_step'],d['roofline']['frac'],d.get('gpu_launches'))"
done
tail -3 gpurun_out/fuse_gputest.log
