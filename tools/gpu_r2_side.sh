#!/bin/bash
# A/B: CTA cap of the GEMMs on the weight-gradient side streams (NASPIPE_SIDE_SMS)
cd "$(dirname "$0")/.."
O=gpurun_out/side; mkdir -p $O
A="--steps 40 --warmup 5 --no-secondary --no-cpu --no-e2e --no-repro"
for wl in spos transformer; do
  for cap in 0 128 100 74 0 128 100 74; do
    NASPIPE_SIDE_SMS=$cap timeout 300 python bench.py --workload $wl $A > $O/${wl}_$cap.json 2>>$O/err.log
    python -c "import json;d=json.loads(open('$O/${wl}_$cap.json').read().strip().splitlines()[-1]);print('$wl cap=$cap',round(d['value'],1),round(d['ms_per_step'],3),round(d['roofline']['frac'],3))"
  done
done
