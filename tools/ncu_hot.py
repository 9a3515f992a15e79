"""Hottest SASS instructions (stall samples) of one kernel of an ncu report.
Usage: ncu_hot.py report.ncu-rep kernel_regex [N]"""
import csv, subprocess, sys
rep, kre = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", "regex:" + kre,
                      "--launch-count", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hi = next(i for i, r in enumerate(rows) if "Address" in r)
h = rows[hi]
it, isrc, iex = h.index("Warp Stall Sampling (All Samples)"), h.index("Source"), h.index("Instructions Executed")
recs = []
for r in rows[hi + 1:]:
    if len(r) != len(h):
        continue
    try:
        recs.append((int(r[it] or 0), r[isrc].strip(), r[iex]))
    except ValueError:
        continue
tot = sum(x[0] for x in recs) or 1
print("total samples", tot)
for s, src, ex in sorted(recs, reverse=True)[:n]:
    print(f"{s / tot:.3f} {ex:>9} {src[:100]}")
