#!/bin/bash
# second one-knob-at-a-time sweep (configs[1] elementwise/split-K knobs, configs[2] knobs)
cd "$(dirname "$0")/.."
O=gpurun_out/sweep2; mkdir -p $O
A="--steps 40 --warmup 5 --no-secondary --no-cpu --no-e2e --no-repro"
run() {
  local lab=$1; shift
  env "$@" timeout 300 python bench.py $WL $A > $O/$lab.json 2>>$O/err.log
  python -c "import json;d=json.loads(open('$O/$lab.json').read().strip().splitlines()[-1]);print('$lab',round(d['ms_per_step'],4),round(d['roofline']['frac'],4))"
}
for rep in 1 2; do
  WL=""
  run spos_base_$rep
  run spos_ewwaves2_$rep NASPIPE_EW_WAVES=2
  run spos_gswaves2_$rep NASPIPE_GS_WAVES=2
  run spos_splitk8_$rep NASPIPE_SPLITK_CTAS_PER_SM=8
  run spos_dwtw32_$rep NASPIPE_DW_TW=32
  WL="--workload transformer"
  run tf_base_$rep
  run tf_lnrows8_$rep NASPIPE_LN_ROWS=8
  run tf_csrows32_$rep NASPIPE_CS_ROWS=32
  run tf_nopair_$rep NASPIPE_GEMM_PAIR=0
  run tf_splitk8_$rep NASPIPE_SPLITK_CTAS_PER_SM=8
done
