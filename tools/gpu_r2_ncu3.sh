#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
timeout 600 $NCU --set full --import-source on --clock-control none -k regex:"bn_apply_kernel|bn_bwd_apply_kernel|bn_bwd_reduce_kernel" -s 200 -c 9 -o gpurun_out/ncu_bn -f python tools/kernel_table.py spos 2 > gpurun_out/ncu_bn.log 2>&1; echo bn=$?
timeout 600 $NCU --set full --import-source on --clock-control none -k regex:"attn_bwd_tc|attn_fwd_tc" -s 20 -c 4 -o gpurun_out/ncu_attn -f python tools/kernel_table.py transformer 1 > gpurun_out/ncu_attn.log 2>&1; echo attn=$?
timeout 600 $NCU --set full --import-source on --clock-control none -k regex:"dw_dgrad_s2" -s 4 -c 3 -o gpurun_out/ncu_s2 -f python tools/kernel_table.py spos 2 > gpurun_out/ncu_s2.log 2>&1; echo s2=$?
ls -la gpurun_out/*.ncu-rep
