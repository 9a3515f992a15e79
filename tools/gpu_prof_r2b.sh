#!/bin/bash
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIfLb0 -s 1 -c 1 -o gpurun_out/prof_wf32_r2s \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIdLb0 -s 1 -c 1 -o gpurun_out/prof_wf64_r2s \
    python bench.py --workload C3 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/ncu_full64.log 2>&1
tail -1 gpurun_out/ncu_full64.log
for wl in C2 C3; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$wl.csv \
    python bench.py --workload $wl --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
