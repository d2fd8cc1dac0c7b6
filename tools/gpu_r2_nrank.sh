#!/bin/bash
# the N > 1 bench path (torchrun, peer transport, max-over-ranks timing, bit_repro vs D = 1)
# with both ranks sharing the box's one GPU
export NASPIPE_BENCH_SHARE_GPU=1
for w in spos transformer; do
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --workload $w --gpus 2 --steps 10 --warmup 3 --no-cpu --no-secondary > gpurun_out/r2_bench_n2_$w.json 2> gpurun_out/r2_bench_n2_$w.err
echo "$w rc=$?"
tail -c 1500 gpurun_out/r2_bench_n2_$w.json; echo
grep -i -E "error|Traceback" gpurun_out/r2_bench_n2_$w.err | head -5
done
