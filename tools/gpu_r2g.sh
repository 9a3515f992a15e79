#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
WL="C2 C3" timeout 900 bash tools/ab_r2.sh ab_libs/libphmm_cur.so paper_conf_ipps_wangxc17_b200/libphmm.so 2>&1 | tee gpurun_out/ab13.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C2.csv \
    python bench.py --workload C2 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_shares.py gpurun_out/launches_C2.csv 2>/dev/null | head -12
