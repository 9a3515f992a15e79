#!/bin/bash
# ncu --set full of the preparation kernels of one C2 call (and of C3's table builds):
# where their time goes against HBM bandwidth
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:k_build_table_wf|k_alloc_blocks_wf|k_hap_codes_wf|k_pair_bins|k_validate|k_scan_bins" -s 0 -c 8 \
    -o gpurun_out/prof_prep_c2 python bench.py --steps 1 --warmup 0 --profile-steps --no-e2e --no-cpu-baseline --no-extra > gpurun_out/prof_prep.log 2>&1
tail -2 gpurun_out/prof_prep.log
python tools/ncu_summary.py gpurun_out/prof_prep_c2.ncu-rep gpu__time_duration.sum dram__bytes_read.sum dram__bytes_write.sum \
    dram__throughput.avg.pct_of_peak_sustained_elapsed sm__warps_active.avg.pct smsp__issue_active.avg.pct \
    launch__grid_size launch__registers_per_thread lts__t_sectors_op_write.sum l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum \
    smsp__average_warp_latency_issue_stalled_long_scoreboard smsp__pcsamp_warps_issue_stalled_long_scoreboard \
    > gpurun_out/prep_summary.txt 2>&1
python tools/ncu_stalls.py gpurun_out/prof_prep_c2.ncu-rep > gpurun_out/prep_stalls.txt 2>&1
