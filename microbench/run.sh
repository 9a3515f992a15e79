#!/bin/bash
# Runs the issue-rate microbenchmarks on the GPU box; output -> gpurun_out/micro.jsonl
set -e
cd "$(dirname "$0")"
mkdir -p ../gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv | tee ../gpurun_out/micro_clocks.txt
./issue_rates | tee ../gpurun_out/micro.jsonl
