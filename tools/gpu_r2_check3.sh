# round-2 GPU check 3: full GPU suite, default bench, ncu launch list of one bench step
set -x
timeout 1500 python -m pytest tests -m gpu -q -s -p no:cacheprovider > gpurun_out/r2_gputest3.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed" gpurun_out/r2_gputest3.log | tail -3
grep -E "^FAILED" gpurun_out/r2_gputest3.log | head -20
timeout 900 python bench.py > gpurun_out/r2_bench3.json 2> gpurun_out/r2_bench3.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench3.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches']/d['steps'],d['fractions'])"
