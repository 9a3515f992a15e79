"""Shared-memory bank-conflict evidence of an ncu report: the l1tex conflict counters and,
per SASS instruction, actual vs ideal shared wavefronts (excess = bank conflicts).
Usage: ncu_banks.py report.ncu-rep"""
import csv
import subprocess
import sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(raw.splitlines()))
H, U, V = rr[0], rr[1], rr[2]
print(f"# {rep}: {V[H.index('Kernel Name')][:60]}")
for w in ["gpu__time_duration.sum", "launch__registers_per_thread", "launch__block_size", "launch__grid_size",
          "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
          "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
          "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
          "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
          "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum"]:
    if w in H:
        print(f"{w} = {V[H.index(w)]} {U[H.index(w)]}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hi = [i for i, r in enumerate(rows[:3]) if "Address" in r][0]
h = rows[hi]
iw, ii = h.index("L1 Wavefronts Shared"), h.index("L1 Wavefronts Shared Ideal")
tot = ideal = 0
worst = []
for r in rows[hi + 1:]:
    if len(r) != len(h):
        continue
    try:
        w, d = int(r[iw] or 0), int(r[ii] or 0)
    except ValueError:
        continue
    tot += w
    ideal += d
    if w > d:
        worst.append((w - d, r[h.index("Source")].strip()[:60]))
print(f"\n# per-instruction shared wavefronts (ncu source page): actual {tot}, ideal {ideal}, excess {tot - ideal}")
for x, s in sorted(worst, reverse=True)[:10]:
    print(f"  excess {x:>10}  {s}")
# by opcode
from collections import defaultdict
act, exc = defaultdict(int), defaultdict(int)
isrc = h.index("Source")
for r in rows[hi + 1:]:
    if len(r) != len(h):
        continue
    try:
        w, d = int(r[iw] or 0), int(r[ii] or 0)
    except ValueError:
        continue
    if not w:
        continue
    t = r[isrc].strip().split()
    op = (t[1] if t and t[0].startswith("@") and len(t) > 1 else (t[0] if t else "?")).split(".")[0]
    act[op] += w
    exc[op] += w - d
print("\n# by opcode: actual / excess shared wavefronts")
for op in sorted(act, key=lambda k: -act[k]):
    print(f"  {op:8s} {act[op]:>12,} / {exc[op]:>10,}")
