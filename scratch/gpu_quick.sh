#!/bin/bash
# parity tests + bench + launch list + ncu on the FP32 wavefront kernel
mkdir -p gpurun_out
python -m pytest tests/test_gpu_parity.py -x -q -m gpu 2>&1 | tail -4
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
ncu --set full --clock-control none --import-source on -k regex:k_wavefront_f32 -s 1 -c 1 -o gpurun_out/prof_wf32 python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
