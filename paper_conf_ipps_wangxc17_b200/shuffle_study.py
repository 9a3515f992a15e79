"""The paper's own experiment re-run on sm_100a.

1. Instruction-latency microbenchmarks (Listing 1, L14@19, §II-B): one dependent
   chain per kernel, timed over ten iteration counts; a least-squares line
       t = #iterations * k + beta                 (Eq. 1 / Eq. 2, k = latency_x + alpha)
   gives the slope k of each kernel, and
       latency_shfl      = latency_reg + k_shfl - k_reg                      (from Eq. 1-2)
       latency_sharedmem = latency_reg + k_sharedmem - k_reg                 (Eq. 3)
       latency_sync      = latency_reg + k_sync - k_reg - latency_sharedmem  (Eq. 4)
   with latency_reg = 1 ("register access takes one cycle", L14@3560).
2. Performance model (§IV-D, L22@1543 / L22@1832):
       performance = parallelism * frequency / latency                     (Eq. 8)
       parallelism = #SM * min(#reg/SM / #reg/thread,
                               #smem/SM / #smem/block * threads/block)     (Eq. 7)
   instantiated for B200 and for the two exchange designs of our wavefront kernel:
   design B (shuffle, libphmm.so) and design A (shared-memory line buffer,
   libphmm_xsmem.so, Listing 2a L20@44), as the paper's Table II/III validation
   (L24@2660) does for PH1/PH2.

The arithmetic here (regression, Eq. 1-4, Eq. 7-8) is host logic, tested on CPU
(tests/test_shuffle_study.py); `run_microbenchmarks` and `main` need the GPU.
This module is a measurement tool: it is not on the PairHMM path and does not touch
oracle/.
"""
from __future__ import annotations

import ctypes
import json
import os
import subprocess
import sys
from dataclasses import asdict, dataclass, field
from typing import Dict, List, Optional, Sequence

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(_PKG)

LATENCY_REG = 1.0  # cycles, the paper's assumption (L14@3560)
ITERATIONS = tuple(range(1000, 11000, 1000))  # "ten runs with different values of ITERATIONS"

KIND = {"reg": 0, "shfl_idx": 1, "shfl_up": 2, "shfl_down": 3, "shfl_xor": 4, "sharedmem": 5,
        "sharedmemsync": 6, "sharedmemsyncwarp": 7}


# ---------------------------------------------------------------- Eq. 1-4
def fit_line(iterations: Sequence[float], t: Sequence[float]):
    """Least-squares t = k * iterations + beta (Eq. 1/2). Returns (k, beta, r2)."""
    x = np.asarray(iterations, dtype=np.float64)
    y = np.asarray(t, dtype=np.float64)
    if x.size < 2 or np.ptp(x) == 0:
        raise ValueError("need at least two distinct iteration counts")
    k, beta = np.polyfit(x, y, 1)
    yhat = k * x + beta
    ss_res = float(np.sum((y - yhat) ** 2))
    ss_tot = float(np.sum((y - y.mean()) ** 2))
    r2 = 1.0 - ss_res / ss_tot if ss_tot > 0 else 1.0
    return float(k), float(beta), r2


def latency_from_slopes(k_x: float, k_reg: float, latency_reg: float = LATENCY_REG) -> float:
    """latency_x = latency_reg + k_x - k_reg (shuffle: Eq. 1-2; shared memory: Eq. 3)."""
    return latency_reg + k_x - k_reg


def sync_latency(k_sync: float, k_reg: float, latency_sharedmem: float, latency_reg: float = LATENCY_REG) -> float:
    """latency_sync = latency_reg + k_sync - k_reg - latency_sharedmem (Eq. 4)."""
    return latency_reg + k_sync - k_reg - latency_sharedmem


def derive_latencies(slopes: Dict[str, float], latency_reg: float = LATENCY_REG) -> Dict[str, float]:
    """All Eq. 1-4 latencies from the fitted slopes {name: k}. 'reg' is required; every
    shuffle variant and 'sharedmem' map through Eq. 1-3, names starting with
    'sharedmemsync' through Eq. 4 (needs 'sharedmem')."""
    k_reg = slopes["reg"]
    out = {"reg": latency_reg}
    for name, k in slopes.items():
        if name == "reg" or name.startswith("sharedmemsync"):
            continue
        out[name] = latency_from_slopes(k, k_reg, latency_reg)
    for name, k in slopes.items():
        if name.startswith("sharedmemsync"):
            out[name] = sync_latency(k, k_reg, out["sharedmem"], latency_reg)
    return out


# ---------------------------------------------------------------- Eq. 7-8
@dataclass
class Platform:
    n_sm: int = 148
    regs_per_sm: int = 65536
    smem_per_sm: int = 233472  # bytes (228 KB)
    threads_per_sm: int = 2048
    freq_hz: float = 1.965e9


@dataclass
class KernelChar:
    name: str
    regs_per_thread: int
    smem_per_block: int  # bytes
    threads_per_block: int
    cells_per_thread_iter: int = 1  # cells one thread updates per iteration


def parallelism_eq7(p: Platform, k: KernelChar) -> float:
    """Eq. 7 as printed: #SM * min(#reg/SM / #reg/thread, #smem/SM / #smem/block * threads/block)."""
    by_reg = p.regs_per_sm / k.regs_per_thread
    by_smem = (p.smem_per_sm / k.smem_per_block) * k.threads_per_block if k.smem_per_block > 0 else float("inf")
    return p.n_sm * min(by_reg, by_smem)


def parallelism_resident(p: Platform, k: KernelChar, reg_alloc_unit: int = 256, smem_reserved: int = 1024) -> int:
    """Eq. 7 with the hardware's granularity (whole blocks, register allocation per warp in
    units of 256, 1 KB reserved shared memory per block, the 2048-thread limit): the
    resident threads the occupancy calculator reports. (Extension.)"""
    warps = -(-k.threads_per_block // 32)
    regs_per_warp = -(-k.regs_per_thread * 32 // reg_alloc_unit) * reg_alloc_unit
    blocks_reg = p.regs_per_sm // (regs_per_warp * warps)
    blocks_smem = p.smem_per_sm // (k.smem_per_block + smem_reserved) if k.smem_per_block > 0 else 1 << 30
    blocks_thr = p.threads_per_sm // k.threads_per_block
    return p.n_sm * min(blocks_reg, blocks_smem, blocks_thr) * k.threads_per_block


def performance_eq8(parallelism: float, freq_hz: float, latency_cycles: float, cells_per_thread_iter: int = 1) -> float:
    """Eq. 8: cell updates per second = parallelism * frequency / latency, generalised to
    threads that update several cells per iteration (PH2 updates 4, L26@560)."""
    return parallelism * cells_per_thread_iter * freq_hz / latency_cycles


def implied_latency(perf_cups: float, parallelism: float, freq_hz: float, cells_per_thread_iter: int = 1) -> float:
    """Eq. 8 solved for the iteration latency, from a measured performance (§V-C)."""
    return parallelism * cells_per_thread_iter * freq_hz / perf_cups


@dataclass
class StepCost:
    """Per-iteration cost of one warp of our wavefront kernel (one step = 2K cells per
    lane), from the SASS of its hot loop (tools/sass_loop.py)."""
    instructions: float        # issued warp instructions per step
    fma_pipe_cycles: float     # FMA-pipe cycles per step (FFMA2/FMUL2/FADD2 = 2, FMUL/IMAD = 1)
    critical_path: float       # dependent-chain latency per step (cycles)
    warps_per_scheduler: float


def latency_throughput_aware(c: StepCost) -> float:
    """B200 extension of the paper's latency term: a warp's step takes at least its
    critical path, and at least the issue slots / FMA-pipe cycles of all warps sharing its
    scheduler (the paper's model assumes the critical path alone binds)."""
    return max(c.critical_path, c.warps_per_scheduler * c.instructions, c.warps_per_scheduler * c.fma_pipe_cycles)


# ---------------------------------------------------------------- GPU runner
@dataclass
class MicroResult:
    name: str
    kind: str
    param: int
    threads: int
    iterations: List[int]
    cycles: List[int]
    slope: float = 0.0
    beta: float = 0.0
    r2: float = 0.0


def _lib():
    path = os.path.join(_PKG, "liblatency.so")
    if not os.path.exists(path):
        raise RuntimeError(f"{path} not built (paper_conf_ipps_wangxc17_b200.build.build_latency())")
    L = ctypes.CDLL(path)
    L.phmm_lat_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                               ctypes.c_void_p, ctypes.POINTER(ctypes.c_longlong)]
    L.phmm_lat_run.restype = ctypes.c_int
    return L


def microbenchmark_plan() -> List[tuple]:
    """(name, kind, param, threads): Listing 1's kernels and Fig. 1's shuffle variants."""
    plan = [("reg", "reg", 0, 32), ("shfl_idx_random", "shfl_idx", 0, 32)]
    for d in (1, 2, 4, 8, 16):
        plan += [(f"shfl_up_{d}", "shfl_up", d, 32), (f"shfl_down_{d}", "shfl_down", d, 32),
                 (f"shfl_xor_{d}", "shfl_xor", d, 32)]
    plan += [("sharedmem", "sharedmem", 0, 1)]
    for t in (1, 32, 128, 1024):
        plan += [(f"sharedmemsync_{t}", "sharedmemsync", 0, t)]
    plan += [("sharedmemsyncwarp_32", "sharedmemsyncwarp", 0, 32)]
    return plan


def run_microbenchmarks(iterations: Sequence[int] = ITERATIONS, repeats: int = 3, seed: int = 0) -> List[MicroResult]:
    import torch

    L = _lib()
    rng = np.random.default_rng(seed)
    # chain start values: lane indices (so the pointer chase visits buf[ind] = ind)
    vals = torch.tensor(np.arange(32, dtype=np.float32) * 0 + 1.0, device="cuda")
    chase = torch.tensor(np.arange(32, dtype=np.float32), device="cuda")
    src = torch.tensor(rng.integers(0, 32, size=32).astype(np.int32), device="cuda")
    out = []
    for name, kind, param, threads in microbenchmark_plan():
        inp = chase if kind.startswith("sharedmem") else vals
        cyc = []
        for it in iterations:
            best = None
            for _ in range(repeats):
                c = ctypes.c_longlong(0)
                rc = L.phmm_lat_run(KIND[kind], param, int(it), threads, ctypes.c_void_p(inp.data_ptr()),
                                    ctypes.c_void_p(src.data_ptr()), ctypes.byref(c))
                if rc != 0:
                    raise RuntimeError(f"phmm_lat_run({name}) failed: cudaError {rc}")
                best = c.value if best is None else min(best, c.value)
            cyc.append(int(best))
        r = MicroResult(name, kind, param, threads, list(map(int, iterations)), cyc)
        r.slope, r.beta, r.r2 = fit_line(r.iterations, r.cycles)
        out.append(r)
    return out


def latency_table(results: Sequence[MicroResult]) -> Dict[str, float]:
    slopes = {r.name: r.slope for r in results}
    return derive_latencies(slopes)


# the short-row FP32 wavefront kernel, k_wavefront<float, false> (csrc/wavefront.cuh)
WF32_SYMBOL = "_ZN4phmm11k_wavefrontIfLb0EEEvNS_7WfArgs2IT_EE"


def hot_loop_mix(so_path: str, mangled: str) -> Dict[str, int]:
    """Opcode counts of the innermost loop with the most packed FP32 instructions of a
    kernel (cuobjdump -sass), i.e. one group of 4 steps of the wavefront kernel."""
    import re
    from collections import Counter

    out = subprocess.run(["cuobjdump", "-sass", so_path], capture_output=True, text=True).stdout
    body = [f for f in re.split(r"\n\s+Function : ", out) if f.startswith(mangled)][0]
    ins = []
    for l in body.split("\n"):
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", l)
        if m:
            ins.append((int(m.group(1), 16), m.group(2).strip()))
    loops = []
    for a, t in ins:
        m = re.search(r"BRA\S*\s+(?:\S+,\s*)?(0x[0-9a-f]+)", t)
        if m and int(m.group(1), 16) <= a:
            loops.append((int(m.group(1), 16), a))

    def mix(lo, hi):
        c = Counter()
        for a, t in ins:
            if lo <= a <= hi:
                op = t.split()[1] if t.startswith("@") else t.split()[0]
                c[op.split(".")[0]] += 1
        return c

    best = max(loops, key=lambda l: (mix(*l)["FFMA2"] + mix(*l)["FMUL2"], -(l[1] - l[0])))
    return dict(mix(*best))


def step_cost(mix: Dict[str, int], steps_per_loop: int = 4, warps_per_scheduler: float = 2.0,
              critical_path: float = 0.0) -> StepCost:
    n = sum(mix.values())
    packed = mix.get("FFMA2", 0) + mix.get("FMUL2", 0) + mix.get("FADD2", 0)
    scalar = mix.get("FFMA", 0) + mix.get("FMUL", 0) + mix.get("FADD", 0) + mix.get("IMAD", 0)
    return StepCost(instructions=n / steps_per_loop, fma_pipe_cycles=(2 * packed + scalar) / steps_per_loop,
                    critical_path=critical_path, warps_per_scheduler=warps_per_scheduler)


def critical_path(lat: Dict[str, float], k_fma: float, design: str, K: int = 8) -> float:
    """Latency of one step's dependent chain (paper's LOAD -> COMPUTE -> WRITE view,
    L22@2294): the exchange of the last row (design B: one SHFL + the lane-31 select;
    design A: shared-memory write, __syncwarp, read, __syncwarp), then the K-deep
    I(i,j) = eps*I(i-1,j) + delta*M(i-1,j) chain down the block, whose end feeds the next
    exchange. k_fma = slope of the dependent-FMUL chain (reg kernel)."""
    chain = (K + 1) * k_fma
    if design == "B":
        return lat["shfl_idx_random"] + k_fma + chain
    sw = lat.get("sharedmemsyncwarp_32", 0.0)
    return lat["sharedmem"] + 2 * sw + lat["sharedmem"] + chain


def model_report(doc: dict) -> dict:
    """Eq. 7-8 for design B and design A on B200, validated as in §V-C (L24@2660):
    implied latency from the measured GCUPS vs the latency predicted from the
    microbenchmarks (paper's critical-path view) and from a throughput-aware extension."""
    lat = doc["latency_cycles_eq1_4"]
    k_fma = [m["slope"] for m in doc["microbenchmarks"] if m["name"] == "reg"][0]
    p = Platform(**doc["platform"])
    rep = {}
    for tag, d in doc["designs"].items():
        design = "B" if tag.startswith("B") else "A"
        smem_block = d["smem_per_block"]
        kc = KernelChar(tag, d["regs_per_thread"], smem_block, 128, cells_per_thread_iter=16)
        par7 = parallelism_eq7(p, kc)
        par = parallelism_resident(p, kc)
        perf = d["kernel_gcups"] * 1e9
        f = (d.get("sm_mhz") or p.freq_hz / 1e6) * 1e6
        lat_impl = implied_latency(perf, par, f, 16)
        cp = critical_path(lat, k_fma, design)
        sc = step_cost(d["hot_loop_mix"], critical_path=cp, warps_per_scheduler=par / p.n_sm / 32 / 4)
        lat_tp = latency_throughput_aware(sc)
        rep[tag] = {"parallelism_eq7": par7, "parallelism_resident": par, "implied_latency_cycles": lat_impl,
                    "critical_path_cycles": cp, "instr_per_step": sc.instructions,
                    "fma_pipe_cycles_per_step": sc.fma_pipe_cycles,
                    "predicted_latency_paper": cp, "predicted_gcups_paper": performance_eq8(par, f, cp, 16) / 1e9,
                    "predicted_latency_throughput_aware": lat_tp,
                    "predicted_gcups_throughput_aware": performance_eq8(par, f, lat_tp, 16) / 1e9,
                    "measured_gcups": d["kernel_gcups"],
                    "error_paper": (performance_eq8(par, f, cp, 16) - perf) / perf,
                    "error_throughput_aware": (performance_eq8(par, f, lat_tp, 16) - perf) / perf}
    if "A_smem_line_buffer" in rep and "B_shuffle" in rep:
        a, b = rep["A_smem_line_buffer"], rep["B_shuffle"]
        meas = a["implied_latency_cycles"] - b["implied_latency_cycles"]
        pred = a["critical_path_cycles"] - b["critical_path_cycles"]
        rep["reduction_A_to_B"] = {"measured_cycles": meas, "predicted_cycles_critical_path": pred,
                                   "relative_error": (pred - meas) / meas if meas else None,
                                   "speedup_B_over_A": b["measured_gcups"] / a["measured_gcups"]}
    return rep


def _ptxas_regs(ptxas_txt: str, mangled: str) -> Optional[int]:
    lines = open(ptxas_txt).read().splitlines()
    for i, l in enumerate(lines):
        if mangled in l and "Compiling entry function" in l:
            for l2 in lines[i + 1:i + 6]:
                if "Used" in l2 and "registers" in l2:
                    return int(l2.split("Used")[1].split("registers")[0])
    return None


def _bench_kernel(lib: str, workload: str = "C2") -> dict:
    env = dict(os.environ, PHMM_LIB=lib)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "5", "--warmup", "3", "--no-e2e",
           "--no-cpu-baseline", "--workload", workload]
    res = subprocess.run(cmd, capture_output=True, text=True, env=env, cwd=ROOT)
    if res.returncode != 0:
        raise RuntimeError(res.stderr[-2000:])
    return json.loads(res.stdout.strip().splitlines()[-1])


def main(out_path: str = os.path.join(ROOT, "profiles", "r02_shuffle_study.json")) -> dict:
    """Run the microbenchmarks, bench design B (libphmm.so) and design A
    (libphmm_xsmem.so) on C2, and instantiate Eq. 7-8 for both."""
    import torch

    res = run_microbenchmarks()
    lat = latency_table(res)
    props = torch.cuda.get_device_properties(0)
    plat = Platform(n_sm=props.multi_processor_count)
    designs = {}
    for tag, lib in (("B_shuffle", os.path.join(_PKG, "libphmm.so")),
                     ("A_smem_line_buffer", os.path.join(_PKG, "libphmm_xsmem.so"))):
        b = _bench_kernel(lib)
        r = b["roofline"]
        ptx = os.path.join(_PKG, "ptxas_info.txt") if tag.startswith("B") else lib + ".ptxas.txt"
        mangled = WF32_SYMBOL
        regs = _ptxas_regs(ptx, mangled) or 0
        # C2: N = 300 -> ncols 304, P = 304 + 8 + 4 = 316 (staged switch), ring 320 + 4 slots of 16 B
        ncols = 304
        # wf_warp_smem<float>: prior tables + staging slots (8 x 144 B) + ring (+ design A's line
        # buffer) + the stream's first block
        smem_block = 4 * ((2 * 6 * 2 * 32 * 16 + 8 * 144 + (324 + (32 if tag.startswith("A") else 0)) * 16 + 32 + 15)
                          & ~15)
        designs[tag] = {"lib": os.path.relpath(lib, ROOT), "kernel_gcups": r["achieved"], "frac": r["frac"],
                        "wavefront_ms": r["wavefront_ms"], "step_gcups": b["value"], "regs_per_thread": regs,
                        "smem_per_block": smem_block, "ncols": ncols,
                        "sm_mhz": b.get("clocks", {}).get("sm_mhz"), "hot_loop_mix": hot_loop_mix(lib, mangled)}
    doc = {"platform": asdict(plat), "device": props.name,
           "microbenchmarks": [asdict(r) for r in res], "latency_cycles_eq1_4": lat, "designs": designs}
    doc["model"] = model_report(doc)
    os.makedirs(os.path.dirname(out_path), exist_ok=True)
    with open(out_path, "w") as f:
        json.dump(doc, f, indent=1)
    return doc


if __name__ == "__main__":
    d = main(*sys.argv[1:])
    print(json.dumps(d["latency_cycles_eq1_4"], indent=1))
    print(json.dumps(d["designs"], indent=1))
    print(json.dumps(d["model"], indent=1))
