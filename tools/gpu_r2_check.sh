set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q -s -p no:cacheprovider > gpurun_out/r2_gputest1.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/r2_gputest1.log
echo "== pair trigger 40 steps (PDL early triggers in the CTA-pair GEMM)"
NASPIPE_PAIR_TRIGGER=1 timeout -s KILL 150 python bench.py --workload transformer --no-cpu --no-e2e --no-secondary --steps 40 > gpurun_out/r2_pdl_pairtrig.log 2>&1; echo "rc=$?"
tail -2 gpurun_out/r2_pdl_pairtrig.log | cut -c1-300
echo "== c4 probe, PDL forced on under context switching"
NASPIPE_FORCE_PDL=1 timeout -s KILL 240 python tools/c4_probe.py --subnets 14 --no-drain > gpurun_out/r2_pdl_c4.log 2>&1; echo "rc=$?"
tail -4 gpurun_out/r2_pdl_c4.log
