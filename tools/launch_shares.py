"""Per-kernel time per launch and share of an ncu --metrics gpu__time_duration.sum CSV."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
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
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{v / 1e6 / cnt[k]:8.3f} ms/launch {100 * v / s:5.1f}% {cnt[k]:3d}  {k[:80]}")
