#!/bin/bash
# Final round-2 pass on the final code: GPU suite, smoke, default bench, kernel tables.
cd "$(dirname "$0")/.."
O=gpurun_out/r2c; mkdir -p $O
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/gputest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/gputest.log
grep -E "^FAILED" $O/gputest.log | head
timeout 1200 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench rc=$?"
timeout 300 python tools/kernel_table.py spos 10 > $O/ktab_spos.txt 2>&1
timeout 300 python tools/kernel_table.py transformer 6 > $O/ktab_tf.txt 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference rc=$?"
python -c "import json;d=json.loads(open('$O/bench_default.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches']/d['steps'],d['e2e']['value'],d['bit_repro']['bitwise_equal']); print({k:(round(v.get('value'),1),(v.get('roofline') or {}).get('frac')) for k,v in d.get('secondary',{}).items()})"
tail -c 600 $O/bench_reference.json
