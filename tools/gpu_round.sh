#!/bin/bash
# One GPU round: smoke, full bench line, launch list (ncu timing pass), ncu --set full of the
# FP32 and FP64 wavefront kernels (C2), shared-memory bank conflicts on the striped C4 path.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -2 gpurun_out/bench.err; cat gpurun_out/bench.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIfLb0 -s 1 -c 1 -o gpurun_out/prof_wf32 \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIdLb0 -s 1 -c 1 -o gpurun_out/prof_wf64 \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/prof_wf64.log 2>&1
tail -1 gpurun_out/prof_wf64.log
# C4 (1000 x 1500): every bin is in the long-row launch (k_wavefront<float, true>), one launch per step
ncu --clock-control none --kernel-name-base mangled -k regex:k_wavefrontIfLb1 -c 1 --csv --metrics \
l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,\
l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,\
smsp__inst_executed_op_shared_ld.sum,smsp__inst_executed_op_shared_st.sum,smsp__inst_executed_shfl.sum,\
smsp__issue_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,\
sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,gpu__time_duration.sum,\
launch__block_size,launch__grid_size,dram__bytes_read.sum,dram__bytes_write.sum \
  python bench.py --workload C4 --regions 32 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline \
  > gpurun_out/ncu_c4_banks.csv 2> gpurun_out/ncu_c4_banks.err
python bench.py --workload C4 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C4.json 2>/dev/null
for w in C3 C5; do python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$w.json 2>/dev/null; done
python bench_sw.py > gpurun_out/bench_sw.json 2>/dev/null
