#!/bin/bash
# planned vs timing-driven executor (NASPIPE_FLAG_TIMED), one GPU, 1/2/4 stages on it
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/timed
for wl in spos transformer; do
  for vs in 1 2 4; do
    for mode in planned timed; do
      extra=""; [ $mode = timed ] && extra="--timed"
      timeout 600 python bench.py --workload $wl --steps 30 --warmup 4 --virtual-stages $vs $extra --no-secondary --no-cpu --no-repro --no-e2e > gpurun_out/timed/${wl}_vs${vs}_${mode}.json 2>>gpurun_out/timed/err.log
      python -c "import json;d=json.loads(open('gpurun_out/timed/${wl}_vs${vs}_${mode}.json').read().strip().splitlines()[-1]);t=d.get('timed_executor') or {};print('$wl vs=$vs $mode',round(d['value'],1),round(d['ms_per_step'],3),'pred',t.get('predictions'),'/',t.get('backwards'),'hits',t.get('hits'))"
    done
  done
done
