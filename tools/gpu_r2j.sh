#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tee gpurun_out/pytest_gpu.log | tail -3
python -m paper_conf_ipps_wangxc17_b200.shuffle_study gpurun_out/shuffle_study.json > gpurun_out/shuffle.log 2>&1; tail -2 gpurun_out/shuffle.log
WL="C2 C3" timeout 900 bash tools/ab_r2.sh ab_libs/libphmm_cur.so paper_conf_ipps_wangxc17_b200/libphmm.so 2>&1 | tee gpurun_out/ab11.txt
