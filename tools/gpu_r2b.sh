#!/bin/bash
# A/B of FP32 kernel variants + launch list of one C3 step
mkdir -p gpurun_out
WL="C2 C3" bash tools/ab_r2.sh ab_libs/libphmm_base.so ab_libs/libphmm_col1.so ab_libs/libphmm_col1o3.so ab_libs/libphmm_o2.so 2>&1 | tee gpurun_out/ab2.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv \
    python bench.py --workload C3 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_shares.py gpurun_out/launches_c3.csv | head -30
