#!/bin/bash
# dilated depthwise kernels + CV.c3 analog: kernel tests, parity, bench line
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest -q -x tests/test_gpu_spos_kernels.py -k depthwise 2>&1 | tail -5
timeout 1500 python -m pytest -q -x -s tests/test_gpu_spos.py -k "dilated or cv_c3 or tiny_spos_parity or every_candidate or bitwise" 2>&1 | grep -v "^$" | tail -25
timeout 900 python bench.py --workload cv_c3 --steps 20 --warmup 5 --no-cpu --no-secondary > gpurun_out/r2_bench_cvc3.json 2> gpurun_out/r2_bench_cvc3.err
echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench_cvc3.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline'],d['gpu_launches']/d['steps'],d.get('bit_repro'));[print(k) for k in d['kernels_top'][:10]]"
tail -3 gpurun_out/r2_bench_cvc3.err
