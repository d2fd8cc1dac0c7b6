#!/bin/bash
# one-launch BatchNorm backward (cooperative grid barrier): kernel + parity + bitwise + bench
set -x
timeout 300 python -m pytest -q -x tests/test_gpu_spos_kernels.py -k batchnorm 2>&1 | tail -3
timeout 900 python -m pytest -q -x tests/test_gpu_spos.py tests/test_gpu_policies.py tests/test_gpu_multirank.py tests/test_gpu_context.py tests/test_gpu_mirror.py 2>&1 | tail -4
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu --no-secondary --no-e2e > /tmp/b.json 2>/dev/null; echo "bench rc=$?"
python -c "import json;d=json.loads(open('/tmp/b.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['roofline']['achieved'],d['gpu_launches']/d['steps'],d['bit_repro']['bitwise_equal']);[print(k) for k in d['kernels_top'][:8]]"
