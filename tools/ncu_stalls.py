"""Per-SASS-instruction stall samples of an ncu report (source page), top instructions
and per-opcode totals. Usage: ncu_stalls.py report.ncu-rep [N]"""
import csv, subprocess, sys
from collections import Counter, defaultdict
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
ia, isrc, itot = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
recs = []
for r in rows[2:]:
    if len(r) != len(h):
        continue
    d = {c: int(r[h.index(c)] or 0) for c in cols}
    recs.append((int(r[itot] or 0), r[ia][-5:], r[isrc].strip(), d))
tot = sum(x[0] for x in recs)
by = Counter()
byop = defaultdict(Counter)
for t, a, s, d in recs:
    op = s.split()[0] if s else "?"
    if op.startswith("@"):
        op = s.split()[1]
    op = op.split(".")[0]
    for c, v in d.items():
        by[c] += v
        byop[op][c] += v
print("total samples", tot)
print("by reason:", [(c, round(v / tot, 3)) for c, v in by.most_common(10)])
print("by opcode (share of samples, top reasons):")
for op, c in sorted(byop.items(), key=lambda x: -sum(x[1].values()))[:14]:
    s = sum(c.values())
    print(f"  {op:8s} {s/tot:6.3f}  " + " ".join(f"{k[6:]}={v/tot:.3f}" for k, v in c.most_common(4)))
print("top instructions:")
for t, a, s, d in sorted(recs, key=lambda x: -x[0])[:n]:
    top = sorted(d.items(), key=lambda x: -x[1])[:3]
    print(f"  {a} {t/tot:6.3f} {s[:60]:60s} " + " ".join(f"{k[6:]}={v}" for k, v in top))
