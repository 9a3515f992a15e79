#!/bin/bash
# Full-state GPU pass: smoke, every GPU test, the bench line on each config, SW bench,
# and shared-memory bank-conflict / pipe metrics of the FP32 kernel on the striped C4 path.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; tail -c 300 gpurun_out/bench_c2.err
for w in C3 C4 C5; do
  python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
python bench_sw.py > gpurun_out/bench_sw.json 2> gpurun_out/bench_sw.err
ncu --clock-control none -k regex:k_wavefrontIf -c 1 --metrics \
l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,\
l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,\
smsp__inst_executed_op_shared_ld.sum,smsp__inst_executed_op_shared_st.sum,smsp__inst_executed_shfl.sum,\
smsp__issue_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active,\
sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,\
launch__registers_per_thread,gpu__time_duration.sum \
  --csv python bench.py --workload C4 --regions 32 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline \
  > gpurun_out/ncu_c4_banks.csv 2> gpurun_out/ncu_c4_banks.err
tail -5 gpurun_out/ncu_c4_banks.csv
