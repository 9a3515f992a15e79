#!/bin/bash
# all GPU tests (log under gpurun_out/)
mkdir -p gpurun_out
python -m pytest tests -m gpu -q -x ${@} 2>&1 | tee gpurun_out/pytest_gpu.log | tail -15
