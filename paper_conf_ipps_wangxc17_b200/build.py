"""Builds libphmm.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels
with the repo snapshot to the GPU box)."""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libphmm.so")
SOURCES = [os.path.join(CSRC, "phmm_lib.cu"), os.path.join(CSRC, "wf.cu"), os.path.join(CSRC, "wf_long32.cu"),
           os.path.join(CSRC, "wf_f64.cu")]
# per-source extra flags: the FP32 short-row and the FP64 wavefront kernels are faster with
# ptxas -O1, the FP32 long-row kernel with the default -O3
SOURCE_FLAGS = {"wf.cu": ["-Xptxas", "-O1"]}
def _deps():
    return SOURCES + [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".cuh", ".h"))] + \
        [os.path.join(ROOT, "include", "phmm.h"), os.path.abspath(__file__)]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC",
    "-Xptxas", "-v",
]


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if cand and (os.path.sep not in cand or os.path.exists(cand)):
            return cand
    return "nvcc"


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in _deps())


LATENCY_LIB = os.path.join(PKG, "liblatency.so")
LATENCY_SRC = os.path.join(CSRC, "latency.cu")
# Design-A ablation of the wavefront kernel (row-above exchange through a shared-memory
# line buffer instead of __shfl_sync)
XSMEM_LIB = os.path.join(PKG, "libphmm_xsmem.so")


def build_latency(force: bool = False) -> str:
    """liblatency.so: the paper's Listing 1 latency microbenchmarks (not on the hot path)."""
    if not force and os.path.exists(LATENCY_LIB) and os.path.getmtime(LATENCY_LIB) >= max(
            os.path.getmtime(LATENCY_SRC), os.path.getmtime(os.path.abspath(__file__))):
        return LATENCY_LIB
    tmp = LATENCY_LIB + f".tmp{os.getpid()}"
    cmd = [nvcc(), "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
           "-Xcompiler", "-fPIC", "-shared", "-o", tmp, LATENCY_SRC]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed building liblatency.so")
    os.replace(tmp, LATENCY_LIB)
    return LATENCY_LIB


def build_xsmem(force: bool = False) -> str:
    """libphmm_xsmem.so: libphmm with the shared-memory (design A) row exchange."""
    if not force and os.path.exists(XSMEM_LIB) and os.path.getmtime(XSMEM_LIB) >= max(
            os.path.getmtime(p) for p in _deps()):
        return XSMEM_LIB
    return build(out=XSMEM_LIB, defines=["PHMM_XCHG_SMEM=1"])


SYNTH_LIB = os.path.join(PKG, "libsynth.so")
SYNTH_SRC = os.path.join(CSRC, "synth_gen.c")


def build_synth(force: bool = False) -> str:
    """libsynth.so: the native synthetic batch generator (plain C, OpenMP; not the method)."""
    if not force and os.path.exists(SYNTH_LIB) and os.path.getmtime(SYNTH_LIB) >= os.path.getmtime(SYNTH_SRC):
        return SYNTH_LIB
    tmp = SYNTH_LIB + f".tmp{os.getpid()}"
    res = subprocess.run(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-o", tmp, SYNTH_SRC, "-lm"],
                         capture_output=True, text=True)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("gcc failed building libsynth.so")
    os.replace(tmp, SYNTH_LIB)
    return SYNTH_LIB


def build_all(force: bool = False, verbose: bool = False) -> None:
    build(force=force, verbose=verbose)
    build_synth(force=force)
    build_xsmem(force=force)
    build_latency(force=force)


def build(force: bool = False, verbose: bool = False, out: str = None, defines=(), source_flags=None) -> str:
    """Build libphmm.so (or a variant at ``out`` with extra -D ``defines`` and/or
    per-source flags ``source_flags``, for A/B runs)."""
    sflags = SOURCE_FLAGS if source_flags is None else source_flags
    target = out or LIB
    if not force and out is None and not needs_build():
        return LIB
    tmp = target + f".tmp{os.getpid()}"
    objs, log = [], []
    for src in SOURCES:
        obj = f"{tmp}.{os.path.basename(src)}.o"
        cmd = ([nvcc()] + NVCC_FLAGS + sflags.get(os.path.basename(src), []) + [f"-D{d}" for d in defines]
               + ["-I", os.path.join(ROOT, "include"), "-c", "-o", obj, src])
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0:
            sys.stderr.write(res.stdout + res.stderr)
            raise RuntimeError(f"nvcc failed building {os.path.basename(src)}")
        log.append(res.stderr)
        objs.append(obj)
    res = subprocess.run([nvcc(), "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", tmp] + objs,
                         capture_output=True, text=True)
    for o in objs:
        os.unlink(o)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed linking libphmm.so")
    if verbose:
        sys.stderr.write("".join(log))
    with open(target + ".ptxas.txt" if out else os.path.join(PKG, "ptxas_info.txt"), "w") as f:
        f.write("".join(log))
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    build_all(force="--force" in sys.argv, verbose=True)
    print(LIB)
