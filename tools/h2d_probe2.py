"""H2D copy rates of the pipelined call's job list, replayed with torch copies on one stream
(pinned sources), alone and beside a busy kernel on another stream."""
import sys, os, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_wangxc17_b200 import synth
b = synth.config_batch("C2")
KEYS = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "hap_bases", "pairs")
P = {k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().reshape(-1).view(torch.uint8) for k in KEYS}
D = {k: torch.empty_like(v, device="cuda") for k, v in P.items()}
n = b.n_pairs
bounds = [0, n // 16, n // 8, n // 4, n // 2, n]
ro, ho = b.read_offsets, b.hap_offsets
jobs = []
r0 = h0 = 0
for k in range(5):
    p0, p1 = bounds[k], bounds[k + 1]
    jobs.append(("pairs", 8 * p0, 8 * p1))
    rmax = int(b.pairs[p0:p1, 0].max()) + 1 if k < 4 else b.n_reads
    hmax = int(b.pairs[p0:p1, 1].max()) + 1 if k < 4 else b.n_haps
    r1, h1 = int(ro[rmax]), int(ho[hmax])
    jobs.append(("hap_bases", h0, h1))
    for a in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals"):
        jobs.append((a, r0, r1))
    r0, h0 = r1, h1
def run(busy):
    s = torch.cuda.Stream(); s2 = torch.cuda.Stream()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(len(jobs) + 1)]
    x = torch.randn(8192, 8192, device="cuda")
    torch.cuda.synchronize()
    if busy:
        with torch.cuda.stream(s2):
            for _ in range(20): x = x @ x * 1e-4
    with torch.cuda.stream(s):
        ev[0].record(s)
        for j, (a, lo, hi) in enumerate(jobs):
            D[a][lo:hi].copy_(P[a][lo:hi], non_blocking=True)
            ev[j + 1].record(s)
    torch.cuda.synchronize()
    out = []
    for j, (a, lo, hi) in enumerate(jobs):
        us = ev[j].elapsed_time(ev[j + 1]) * 1e3
        out.append(f"{a[:5]}:{(hi-lo)/1e6:.2f}MB/{us:.0f}us")
    print("busy" if busy else "idle", " ".join(out), flush=True)
run(False); run(False); run(True)
