#!/bin/bash
# round-2 bench lines (default C2 + C3 object; full C5 at N=1), and the ptxas -O2/-O3 builds of
# the wavefront kernels through every GPU parity test
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; tail -c 300 gpurun_out/bench_c2.json
python bench.py --workload C5 --steps 3 --warmup 3 > gpurun_out/bench_c5_full.json 2> gpurun_out/bench_c5_full.err; tail -c 300 gpurun_out/bench_c5_full.json
for v in o3 o2; do echo "== $v"; PHMM_LIB=ab_libs/libphmm_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x 2>&1 | tail -2; done
