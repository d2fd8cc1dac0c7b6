#!/bin/bash
# throughput with V pipeline stages on one GPU (concurrent stage streams)
for w in spos transformer cv_c3 nlp_c3; do
for v in 1 2 4; do
  timeout 600 python bench.py --workload $w --virtual-stages $v --steps 20 --warmup 5 --no-cpu --no-secondary --no-e2e --no-profile --no-repro > /tmp/vs.json 2>/dev/null
  python -c "import json;d=json.loads(open('/tmp/vs.json').read().splitlines()[-1]);print('$w', $v, round(d['value'],1), round(d['ms_per_step'],3))"
done; done
