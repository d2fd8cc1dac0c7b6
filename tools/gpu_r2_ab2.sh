#!/bin/bash
# A/B: stream priorities (NASPIPE_STREAM_PRIO) and BatchNorm elementwise grid floor (NASPIPE_EW_MIN_PIX)
cd "$(dirname "$0")/.."
O=gpurun_out/ab2; mkdir -p $O
A="--steps 40 --warmup 5 --no-secondary --no-cpu --no-e2e --no-repro"
run() {  # label env...
  local lab=$1; shift
  env "$@" timeout 300 python bench.py $WL $A > $O/$lab.json 2>>$O/err.log
  python -c "import json;d=json.loads(open('$O/$lab.json').read().strip().splitlines()[-1]);print('$lab',round(d['value'],1),round(d['ms_per_step'],3),round(d['roofline']['frac'],3))"
}
WL=""
for rep in 1 2; do
  run spos_prio0_pix1_$rep NASPIPE_STREAM_PRIO=0 NASPIPE_EW_MIN_PIX=1
  run spos_prio1_pix1_$rep NASPIPE_STREAM_PRIO=1 NASPIPE_EW_MIN_PIX=1
  run spos_prio1_pix4_$rep NASPIPE_STREAM_PRIO=1 NASPIPE_EW_MIN_PIX=4
  run spos_prio1_pix8_$rep NASPIPE_STREAM_PRIO=1 NASPIPE_EW_MIN_PIX=8
done
WL="--workload transformer"
for rep in 1 2; do
  run tf_prio0_$rep NASPIPE_STREAM_PRIO=0
  run tf_prio1_$rep NASPIPE_STREAM_PRIO=1
done
