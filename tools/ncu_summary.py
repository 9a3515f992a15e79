import csv, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h, u = rows[0], rows[1]
keys = sys.argv[2:] if len(sys.argv) > 2 else None
for v in rows[2:]:
    print("kernel:", v[h.index("Kernel Name")][:80])
    for i, name in enumerate(h):
        if keys is None:
            want = any(k in name for k in ["gpu__time_duration.sum", "smsp__issue_active.avg.pct", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__inst_executed_pipe_fma.avg.pct", "pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct",
              "launch__registers", "launch__occupancy_limit", "dram__bytes_read.sum", "dram__bytes_write.sum", "bank_conflicts_pipe_lsu_mem_shared_op",
              "smsp__inst_executed.sum", "sm__pipe_shared_cycles_active.avg.pct", "launch__grid_size", "smsp__warps_eligible.avg.per_cycle_active",
              "smsp__thread_inst_executed_per_inst_executed.ratio", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "sm__cycles_elapsed.avg.per_second",
              "pipe_fmaheavy", "pipe_fmalite"]) and not name.endswith("_max") and "per_second" not in name or name == "sm__cycles_elapsed.avg.per_second"
        else:
            want = any(k in name for k in keys)
        if want:
            print(f"  {name} = {v[i]} {u[i]}")
