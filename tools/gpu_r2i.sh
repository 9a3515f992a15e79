#!/bin/bash
# round-2 evidence (2): sanitizers on the staged kernels, shuffle study (design A vs B) re-run,
# Smith-Waterman bench + ALU-pipe utilisation of its fill kernel, repeatability of the default line
mkdir -p gpurun_out
bash tools/sanitize.sh 2>&1 | tee gpurun_out/sanitize.txt
python -m paper_conf_ipps_wangxc17_b200.shuffle_study gpurun_out/shuffle_study.json > gpurun_out/shuffle.log 2>&1; tail -3 gpurun_out/shuffle.log
python bench_sw.py > gpurun_out/bench_sw.json 2>/dev/null; tail -c 400 gpurun_out/bench_sw.json
ncu --clock-control none --kernel-name-base mangled -k regex:k_sw_fill -c 1 --csv --metrics \
sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,\
smsp__issue_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,\
smsp__inst_executed.sum,gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread \
  python bench_sw.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_sw.csv 2> gpurun_out/ncu_sw.err
for i in 1 2 3; do python bench.py --no-cpu-baseline > gpurun_out/rep_$i.json 2>/dev/null; done
