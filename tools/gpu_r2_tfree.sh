#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_spos.py tests/test_gpu_spos_kernels.py tests/test_gpu_policies.py tests/test_gpu_mirror.py tests/test_gpu_multirank.py tests/test_gpu_context.py tests/test_gpu_timed.py -x -q > gpurun_out/tfree_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/tfree_tests.log
for t in 0 1 0 1; do
  if [ $t = 1 ]; then export NASPIPE_BN_TICKETS=1; else unset NASPIPE_BN_TICKETS; fi
  timeout 300 python bench.py --steps 40 --warmup 5 --no-secondary --no-cpu --no-e2e > gpurun_out/tfree_b$t.json 2>>gpurun_out/tfree_err.log
  python -c "import json;d=json.loads(open('gpurun_out/tfree_b$t.json').read().strip().splitlines()[-1]);print('tickets=$t',d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches'],d['bit_repro']['bitwise_equal'],d['bit_repro']['runs'][0]['sha256'][:16])"
done
unset NASPIPE_BN_TICKETS
timeout 300 python tools/kernel_table.py spos 10 > gpurun_out/ktab_tfree.txt 2>&1; grep "bn_\|span" gpurun_out/ktab_tfree.txt
