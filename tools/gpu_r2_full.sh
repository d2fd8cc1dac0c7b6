#!/bin/bash
# full GPU suite + smoke + default bench (wall-clock of each)
mkdir -p gpurun_out
t0=$(date +%s)
timeout 3000 python -m pytest tests -m gpu -q -x --durations=25 > gpurun_out/r2_gpu_suite.log 2>&1
echo "suite rc=$? $(( $(date +%s) - t0 ))s"
tail -40 gpurun_out/r2_gpu_suite.log
t0=$(date +%s)
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2_smoke.log 2>&1
echo "smoke rc=$? $(( $(date +%s) - t0 ))s"
tail -3 gpurun_out/r2_smoke.log
t0=$(date +%s)
timeout 1500 python bench.py > gpurun_out/r2_bench_default.json 2> gpurun_out/r2_bench_default.err
echo "bench rc=$? $(( $(date +%s) - t0 ))s"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench_default.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['e2e'],d['clocks'],d['gpu_launches']/d['steps']);print({k:(v.get('value'),v.get('ms_per_step'),v.get('error'),(v.get('roofline') or {}).get('frac')) for k,v in d['secondary'].items()})"
