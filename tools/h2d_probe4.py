"""Does reading a page-locked buffer on several CPU threads right before its H2D copy slow the
copy (DMA reads of lines held in CPU caches)? Copy rate of the pinned pair list after no CPU
read, after a 1-thread read and after an 8-thread read."""
import sys, os, numpy as np, torch
from concurrent.futures import ThreadPoolExecutor
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_wangxc17_b200 import synth
b = synth.config_batch("C2")
pairs_t = torch.from_numpy(np.ascontiguousarray(b.pairs)).pin_memory().reshape(-1)
pn = pairs_t.numpy()
dst = torch.empty_like(pairs_t, device="cuda")
s = torch.cuda.Stream()
pool = ThreadPoolExecutor(8)
def copy_us():
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s); dst.copy_(pairs_t, non_blocking=True); e1.record(s)
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1) * 1e3, 1)
def read1(): int(pn.max())
def read8():
    parts = np.array_split(pn, 8)
    list(pool.map(lambda a: int(a.max()), parts))
def write8():
    parts = np.array_split(pn, 8)
    list(pool.map(lambda a: a.__iadd__(0), parts))
for name, f in [("none", lambda: None), ("read1", read1), ("read8", read8), ("write8", write8), ("none", lambda: None)]:
    r = []
    for _ in range(4):
        f(); r.append(copy_us())
    print(name, r, "us for 8 MB", flush=True)
