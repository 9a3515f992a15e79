#!/bin/bash
# Striped-path evidence: ncu --set full of the FP32 long-row kernel on C4 (1000 x 1500,
# 2 passes of 64 blocks per pair, ring carry + ring rescale), for bank conflicts per instruction.
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIfLb1 -s 1 -c 1 \
    -o gpurun_out/prof_c4_wf32 python bench.py --workload C4 --regions 32 --steps 1 --warmup 1 --profile-steps \
    --no-e2e --no-cpu-baseline > gpurun_out/prof_c4.log 2>&1
tail -1 gpurun_out/prof_c4.log
