#!/bin/bash
# ncu --set full of the FP32 wavefront kernel for a given libphmm variant ($1), report name $2
mkdir -p gpurun_out
PHMM_DEBUG=1 PHMM_LIB=$1 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIf -s 1 -c 1 -o gpurun_out/$2 \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/$2.log 2>&1
tail -1 gpurun_out/$2.log
