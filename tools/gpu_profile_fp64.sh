#!/bin/bash
# ncu --set full of the FP64 (rescue) wavefront kernel on the C2 bench step
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontId -s 1 -c 1 -o gpurun_out/prof_wf64 \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/prof_wf64.log 2>&1
tail -1 gpurun_out/prof_wf64.log
