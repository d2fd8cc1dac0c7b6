#!/bin/bash
# one-knob-at-a-time A/B sweep of the SPOS launch knobs on the final code (configs[1])
cd "$(dirname "$0")/.."
O=gpurun_out/sweep; mkdir -p $O
A="--steps 40 --warmup 5 --no-secondary --no-cpu --no-e2e --no-repro"
run() {
  local lab=$1; shift
  env "$@" timeout 300 python bench.py $A > $O/$lab.json 2>>$O/err.log
  python -c "import json;d=json.loads(open('$O/$lab.json').read().strip().splitlines()[-1]);print('$lab',round(d['ms_per_step'],4),round(d['roofline']['frac'],4))"
}
for rep in 1 2; do
  run base_$rep
  for v in 1 2 4; do run strips${v}_$rep NASPIPE_DW_STRIPS=$v; done
  for v in 148 444; do run redctas${v}_$rep NASPIPE_RED_CTAS=$v; done
  for v in 148 592; do run dwred${v}_$rep NASPIPE_DW_RED_CTAS=$v; done
  run miniters4_$rep NASPIPE_RED_MIN_ITERS=4
  run unroll4_$rep NASPIPE_BN_UNROLL=4
done
