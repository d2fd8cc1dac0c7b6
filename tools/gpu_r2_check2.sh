# round-2 GPU check 2: multi-rank peer transport, new bench, PDL repros (diagnostics)
set -x
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_policies.py -q -s -p no:cacheprovider > gpurun_out/r2_multirank.log 2>&1; echo "multirank rc=$?"
tail -15 gpurun_out/r2_multirank.log
timeout 900 python bench.py > gpurun_out/r2_bench_default.json 2> gpurun_out/r2_bench_default.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/r2_bench_default.json; tail -5 gpurun_out/r2_bench_default.err
for i in 1 2 3; do
  NASPIPE_FORCE_PDL=1 timeout -s KILL 200 python tools/c4_probe.py --subnets 14 --no-drain > gpurun_out/r2_pdl_c4_$i.log 2>&1; echo "c4 pdl run $i rc=$?"; tail -1 gpurun_out/r2_pdl_c4_$i.log
done
NASPIPE_FORCE_PDL=1 timeout 600 python -m pytest tests/test_gpu_context.py -q -p no:cacheprovider > gpurun_out/r2_pdl_context.log 2>&1; echo "context+pdl rc=$?"; tail -2 gpurun_out/r2_pdl_context.log
