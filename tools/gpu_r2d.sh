#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tee gpurun_out/pytest_gpu.log | tail -3
timeout 300 python tools/small_batch.py 1024 > gpurun_out/small_batch.json 2> gpurun_out/small_batch.err; tail -c 1500 gpurun_out/small_batch.json; tail -3 gpurun_out/small_batch.err
python -c "import __graft_entry__ as g; g.smoke()"
