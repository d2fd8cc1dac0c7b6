# round-2 GPU check 4: SPOS family tests + kernels, default bench
set -x
timeout 1200 python -m pytest tests/test_gpu_spos.py tests/test_gpu_spos_kernels.py tests/test_gpu_context.py tests/test_gpu_policies.py -q -s -p no:cacheprovider > gpurun_out/r2_gputest4.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed" gpurun_out/r2_gputest4.log | tail -3
grep -E "^FAILED" gpurun_out/r2_gputest4.log | head -20
timeout 1200 python bench.py > gpurun_out/r2_bench4.json 2> gpurun_out/r2_bench4.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench4.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches']/d['steps'],d['fractions']); [print(k) for k in d['kernels_top']]; print({k:(v.get('value'),v.get('error')) for k,v in d['secondary'].items()})"
