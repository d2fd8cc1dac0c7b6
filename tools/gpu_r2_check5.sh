# round-2 GPU check 5: SPOS tests + kernel unit tests + multirank, default bench
set -x
timeout 1200 python -m pytest tests/test_gpu_spos.py tests/test_gpu_spos_kernels.py tests/test_gpu_policies.py tests/test_gpu_multirank.py -q -s -p no:cacheprovider > gpurun_out/r2_gputest5.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed" gpurun_out/r2_gputest5.log | tail -3
grep -E "^FAILED" gpurun_out/r2_gputest5.log | head -20
timeout 1200 python bench.py --no-secondary > gpurun_out/r2_bench5.json 2> gpurun_out/r2_bench5.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench5.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['gpu_launches']/d['steps'],d['fractions'],d['bit_repro']['bitwise_equal']); [print(k) for k in d['kernels_top']]"
