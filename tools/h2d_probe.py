import sys, os, numpy as np, torch, json
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_wangxc17_b200 import synth
b = synth.config_batch("C2")
KEYS = ("read_bases", "read_offsets", "hap_bases", "pairs")
def t(src, dst, reps=5):
    s = torch.cuda.Stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        dst.copy_(src, non_blocking=True)
        e0.record(s)
        for _ in range(reps): dst.copy_(src, non_blocking=True)
        e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    return round(ms*1e3,1), round(src.numel()*src.element_size()/ms/1e6,1)
for k in KEYS:
    a = torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().reshape(-1)
    d = torch.empty_like(a, device="cuda")
    n = a.numel()
    sl = slice(0, n//16)
    print(k, a.dtype, a.numel()*a.element_size(), "whole us,GB/s", t(a, d), "1/16 slice", t(a[sl], d[sl]), "mid slice", t(a[n//2:n//2+n//16], d[n//2:n//2+n//16]), flush=True)
x = torch.empty(8<<20, dtype=torch.uint8).pin_memory(); dx = torch.empty_like(x, device="cuda")
print("fresh 8MB pinned", t(x, dx))
y = torch.from_numpy(np.ascontiguousarray(b.pairs)).pin_memory()
print("pairs 2D", y.shape, y.is_pinned(), t(y, torch.empty_like(y, device="cuda")))
z = torch.from_numpy(np.ascontiguousarray(b.pairs).astype(np.int32)).pin_memory()
print("pairs astype int32", t(z, torch.empty_like(z, device="cuda")))
# CPU-touch effect: read the pinned buffer on the CPU right before each copy
a = torch.from_numpy(np.ascontiguousarray(b.pairs)).pin_memory().reshape(-1)
d = torch.empty_like(a, device="cuda")
an = a.numpy()
def t_touch(reps=5):
    s = torch.cuda.Stream(); res = []
    for _ in range(reps):
        int(an.max())
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s); d.copy_(a, non_blocking=True); e1.record(s)
        torch.cuda.synchronize(); res.append(e0.elapsed_time(e1))
    return [round(x*1e3,1) for x in res]
print("pairs copy after CPU read (us):", t_touch())
def t_write(reps=5):
    s = torch.cuda.Stream(); res = []
    for _ in range(reps):
        an[::1024] += 0
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s); d.copy_(a, non_blocking=True); e1.record(s)
        torch.cuda.synchronize(); res.append(e0.elapsed_time(e1))
    return [round(x*1e3,1) for x in res]
print("pairs copy after CPU write (us):", t_write())
