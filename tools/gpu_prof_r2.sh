#!/bin/bash
# round-2 evidence: launch lists (C2, C3), ncu --set full of the FP32 kernel (C2), bank-counter
# microbenchmark, small-batch figure, pageable staging probe
mkdir -p gpurun_out
ncu --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__inst_executed_op_shared_st.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum \
    --csv microbench/bank_counter > gpurun_out/bank_counter.csv 2>&1
for wl in C2 C3; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$wl.csv \
    python bench.py --workload $wl --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIfLb0 -s 1 -c 1 -o gpurun_out/prof_wf32_r2 \
    python bench.py --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_wavefrontIdLb0 -s 1 -c 1 -o gpurun_out/prof_wf64_r2 \
    python bench.py --workload C3 --steps 1 --warmup 1 --profile-steps --no-e2e --no-cpu-baseline > gpurun_out/ncu_full64.log 2>&1
tail -1 gpurun_out/ncu_full64.log
timeout 300 python tools/small_batch.py 1024 > gpurun_out/small_batch.json 2> gpurun_out/small_batch.err
timeout 300 python tools/stage_probe.py 8 > gpurun_out/stage_probe.json 2>&1
