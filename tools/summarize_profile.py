"""Summarise an ncu launch list + a full capture into profiles/ (committed evidence).

usage: python tools/summarize_profile.py <tag>   (reads gpurun_out/launches.csv, prof_wf32.ncu-rep, bench.json)
"""
import csv
import json
import subprocess
import sys
from collections import defaultdict

tag = sys.argv[1]
out_dir = "profiles"

# ---- launch list: share of the step per kernel (cold-cache, serialised timings)
rows = list(csv.reader(open("gpurun_out/launches.csv")))
hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
h = rows[hi]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    tot[r[ki]] += float(r[vi].replace(",", ""))
    cnt[r[ki]] += 1
s = sum(tot.values())
with open(f"{out_dir}/{tag}_launches.txt", "w") as f:
    f.write("# ncu --metrics gpu__time_duration.sum --clock-control none, bench.py --steps 2 --warmup 1 (C2)\n")
    f.write("# per-launch times are cold-cache and serialised: compare SHARES, not absolutes\n")
    f.write(f"{'total ms':>10} {'share':>7} {'n':>4}  kernel\n")
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        f.write(f"{v / 1e6:10.3f} {100 * v / s:6.1f}% {cnt[k]:4d}  {k[:110]}\n")

# ---- full capture of the FP32 wavefront kernel
raw = subprocess.run(["ncu", "-i", "gpurun_out/prof_wf32.ncu-rep", "--page", "raw", "--csv"],
                     capture_output=True, text=True).stdout
rr = list(csv.reader(raw.splitlines()))
H, U, V = rr[0], rr[1], rr[2]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__warps_eligible.avg.per_cycle_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed.sum",
        "sm__cycles_elapsed.avg.per_second"]
vals = {}
with open(f"{out_dir}/{tag}_ncu_wavefront_f32.txt", "w") as f:
    f.write("# ncu --set full --clock-control none --import-source on -k regex:k_wavefrontIf (k_wavefront<float>, C2, 1 launch)\n")
    for w in want:
        if w in H:
            i = H.index(w)
            vals[w] = (V[i], U[i])
            f.write(f"{w} = {V[i]} {U[i]}\n")
    f.write("\n# warp stall sampling (all samples)\n")
    st = [(H[i], V[i]) for i in range(len(H)) if H[i].startswith("smsp__pcsamp_warps_issue_stalled")
          and not H[i].endswith("not_issued")]
    for k, v in sorted(st, key=lambda x: -float(x[1].replace(",", "") or 0))[:12]:
        f.write(f"{k} = {v}\n")


def to_bytes(v, u):
    x = float(v.replace(",", ""))
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)


traffic = to_bytes(*vals["dram__bytes_read.sum"]) + to_bytes(*vals["dram__bytes_write.sum"])
json.dump({"kernel": "k_wavefront<float>", "workload": "C2 (bench.py default), one launch",
           "dram_bytes_read_plus_write": traffic, "source": f"profiles/{tag}_ncu_wavefront_f32.txt"},
          open(f"{out_dir}/{tag}_wavefront_traffic.json", "w"), indent=1)
# ---- FP64 rescue kernel capture (if present) and per-opcode stall summaries
import os
for rep, name in (("gpurun_out/prof_wf64.ncu-rep", "k_wavefront<double>"),):
    if not os.path.exists(rep):
        continue
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    H, U, V = rr[0], rr[1], rr[2]
    with open(f"{out_dir}/{tag}_ncu_wavefront_f64.txt", "w") as f:
        f.write(f"# ncu --set full --clock-control none -k regex:k_wavefrontId ({name}, C2 rescue pass, 1 launch)\n")
        for w in want + ["sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
                         "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active"]:
            if w in H:
                i = H.index(w)
                f.write(f"{w} = {V[i]} {U[i]}\n")
for rep, sfx in (("gpurun_out/prof_wf32.ncu-rep", "f32"), ("gpurun_out/prof_wf64.ncu-rep", "f64")):
    if os.path.exists(rep):
        st = subprocess.run([sys.executable, "tools/ncu_stalls.py", rep, "25"], capture_output=True, text=True).stdout
        open(f"{out_dir}/{tag}_stalls_wavefront_{sfx}.txt", "w").write(
            f"# tools/ncu_stalls.py {rep} (warp-stall samples per SASS instruction)\n" + st)
try:
    b = json.load(open("gpurun_out/bench.json"))
    json.dump(b, open(f"{out_dir}/{tag}_bench.json", "w"), indent=1)
except Exception as e:  # noqa: BLE001
    print("no bench.json", e)
print(open(f"{out_dir}/{tag}_ncu_wavefront_f32.txt").read())
print(open(f"{out_dir}/{tag}_launches.txt").read()[:1500])
