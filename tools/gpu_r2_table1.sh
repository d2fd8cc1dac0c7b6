#!/bin/bash
# Table 1's search spaces executed on one B200 (round 2): bench lines per space.
cd "$(dirname "$0")/.."
O=gpurun_out/table1; mkdir -p $O
free -g | head -2
A="--steps 10 --warmup 3 --no-secondary --no-cpu --no-repro --no-e2e"
for wl in cv_c2 cv_c1 nlp_c2 nlp_c1; do
  timeout 900 python bench.py --workload $wl $A > $O/$wl.json 2> $O/$wl.err; echo "$wl rc=$?"
  python -c "import json;d=json.loads(open('$O/$wl.json').read().strip().splitlines()[-1]);print('$wl',round(d['value'],1),round(d['ms_per_step'],3),d['roofline']['frac'])" 2>/dev/null || tail -3 $O/$wl.err
done
timeout 1200 python bench.py --workload nlp_c0 --budget-x 3 $A > $O/nlp_c0_budget3.json 2> $O/nlp_c0_budget3.err; echo "nlp_c0 rc=$?"
python -c "import json;d=json.loads(open('$O/nlp_c0_budget3.json').read().strip().splitlines()[-1]);print('nlp_c0',round(d['value'],1),round(d['ms_per_step'],3),d['roofline']['frac'],d['context_switch'])" 2>/dev/null || tail -3 $O/nlp_c0_budget3.err
