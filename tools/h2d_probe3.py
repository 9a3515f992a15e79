"""Is the slow H2D of the pair list a property of the source buffer? Copy 6 MB slices of
(a) the torch-pinned pairs array, (b) a torch-pinned uint8 buffer, (c) the torch-pinned read
array, on a side stream while the main stream launches a chain of tiny kernels."""
import sys, os, time, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_wangxc17_b200 import synth
b = synth.config_batch("C2")
pairs = torch.from_numpy(np.ascontiguousarray(b.pairs)).pin_memory().reshape(-1).view(torch.uint8)
rbase = torch.from_numpy(np.ascontiguousarray(b.read_bases)).pin_memory()
fresh = torch.empty(8 << 20, dtype=torch.uint8).pin_memory()
dst = torch.empty(16 << 20, dtype=torch.uint8, device="cuda")
x = torch.zeros(1024, device="cuda")
s = torch.cuda.Stream()
def t(src, lo, hi, busy):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s); dst[:hi - lo].copy_(src[lo:hi], non_blocking=True); e1.record(s)
    if busy:
        for _ in range(200): x.add_(1.0)
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1) * 1e3, 1)
for busy in (False, True):
    print("busy" if busy else "idle",
          "pairs[2M:8M]", [t(pairs, 2 << 20, 8 << 20, busy) for _ in range(3)],
          "pairs[0:6M]", [t(pairs, 0, 6 << 20, busy) for _ in range(3)],
          "fresh[2M:8M]", [t(fresh, 2 << 20, 8 << 20, busy) for _ in range(3)],
          "reads[2M:8M]", [t(rbase, 2 << 20, 8 << 20, busy) for _ in range(3)], flush=True)
print("pairs ptr", hex(pairs.data_ptr()), "reads ptr", hex(rbase.data_ptr()), "fresh", hex(fresh.data_ptr()))
