"""Print instruction mix of the basic-block loop that contains the most FP32x2 ops in a kernel."""
import re, subprocess, sys
from collections import Counter
so, fn = sys.argv[1], sys.argv[2]
out = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s+Function : ", out)
body = [f for f in funcs if f.startswith(fn)]
assert body, "function not found"
ins = []
for l in body[0].split("\n"):
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", l)
    if m: ins.append((int(m.group(1), 16), m.group(2).strip()))
# backward branches define loops
loops = []
for a, t in ins:
    m = re.search(r"BRA\S*\s+(?:\S+,\s*)?(0x[0-9a-f]+)", t)
    if m:
        tgt = int(m.group(1), 16)
        if tgt <= a: loops.append((tgt, a))
def mix(lo, hi):
    c = Counter()
    for a, t in ins:
        if lo <= a <= hi:
            op = t.split()[0]
            if op.startswith("@"): op = t.split()[1]
            c[op.split(".")[0]] += 1
    return c
best = max(loops, key=lambda l: (mix(*l)["FFMA2"] + mix(*l)["FMUL2"], -(l[1]-l[0])))
for lo, hi in sorted(loops):
    c = mix(lo, hi)
    print(f"loop {lo:#x}-{hi:#x}: {sum(c.values())} instr, FP2={c['FFMA2']+c['FMUL2']+c['FADD2']} FFMA={c['FFMA']} FMUL={c['FMUL']}")
c = mix(*best)
print("hot loop", hex(best[0]), hex(best[1]), "total", sum(c.values()))
print(c.most_common())
if len(sys.argv) > 3:
    for a, t in ins:
        if best[0] <= a <= best[1]: print(hex(a), t)
