# tcgen05 attention bring-up: kernel tests (bounded), then transformer parity + bench
set -x
timeout -s KILL 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention > gpurun_out/r2_attn_kernel.log 2>&1; echo "attn kernel rc=$?"
tail -25 gpurun_out/r2_attn_kernel.log
timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mirror.py -q -s -p no:cacheprovider > gpurun_out/r2_attn_parity.log 2>&1; echo "parity rc=$?"
grep -E "passed|failed|^FAILED|transformer A15|configs\[2\]" gpurun_out/r2_attn_parity.log | head -20
timeout -s KILL 600 python bench.py --workload transformer --no-cpu --no-secondary > gpurun_out/r2_bench_tf_attn.json 2> gpurun_out/r2_bench_tf_attn.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2_bench_tf_attn.json').read().splitlines()[-1]);print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['fractions']['end_to_end_vs_hardware'],d['bit_repro']['bitwise_equal']); [print(k) for k in d['kernels_top']]"
timeout 900 python -m pytest tests/test_gpu_spos.py -q -s -p no:cacheprovider -k multistep > gpurun_out/r2_spos_multistep.log 2>&1; echo "multistep rc=$?"
grep -E "passed|failed|skipped|configs\[1\] full size" gpurun_out/r2_spos_multistep.log | head
