#!/bin/bash
# NLP op families (A38): parity + regressions + NLP.c3 analog bench line
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest -q -x -s tests/test_gpu_parity.py -k "nlp or tiny_transformer" 2>&1 | grep -v "^$" | tail -25
timeout 900 python bench.py --workload nlp_c3 --steps 10 --warmup 3 --no-cpu --no-secondary > gpurun_out/r2_bench_nlpc3.json 2> gpurun_out/r2_bench_nlpc3.err
echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench_nlpc3.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['fractions'],d['gpu_launches']/d['steps'],d.get('bit_repro'));[print(k) for k in d['kernels_top'][:12]]"
tail -3 gpurun_out/r2_bench_nlpc3.err
