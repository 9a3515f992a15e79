#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_pipeline.py -q -x 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tee gpurun_out/pytest_gpu.log | tail -3
timeout 300 python tools/small_batch.py 1024 > gpurun_out/small_batch.json 2> gpurun_out/small_batch.err; tail -c 1500 gpurun_out/small_batch.json; tail -3 gpurun_out/small_batch.err
WL="C2 C3" timeout 300 bash tools/ab_r2.sh paper_conf_ipps_wangxc17_b200/libphmm.so 2>&1 | tee gpurun_out/ab3.txt
