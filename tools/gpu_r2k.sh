#!/bin/bash
# round-2 bench lines of every config with the final kernels
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; tail -c 200 gpurun_out/bench_c2.json
python bench.py --workload C5 --steps 3 --warmup 3 > gpurun_out/bench_c5_full.json 2> gpurun_out/bench_c5_full.err
for w in C3 C4; do python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$w.json 2>/dev/null; done
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/ref.json 2> gpurun_out/ref.err; cat gpurun_out/ref.json
