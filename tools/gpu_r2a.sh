#!/bin/bash
# round 2: GPU tests, default bench (C2 + C3 object), full C5 at N=1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
nproc >> gpurun_out/gpu.txt
python -m pytest tests -m gpu -q -x 2>&1 | tee gpurun_out/pytest_gpu.log | tail -5
python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
python bench.py --workload C5 --steps 3 --warmup 3 > gpurun_out/bench_c5_full.json 2> gpurun_out/bench_c5_full.err
tail -c 600 gpurun_out/bench_c2.json; tail -c 600 gpurun_out/bench_c5_full.json; tail -3 gpurun_out/bench_c5_full.err
