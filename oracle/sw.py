"""ctypes binding of the plain-C Smith-Waterman oracle (oracle/sw_oracle.c).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py). Shares no code with the CUDA product
path. What is computed is stated, with citations (Eq. 5 at L16@3413), in the C
file's header; the readings R20-R25 are in DESIGN.md §12.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sw_oracle.c")
_LIB = os.path.join(_HERE, "liboracle_sw.so")
_lock = threading.Lock()
_lib = None

BT_STOP = -(2 ** 31)
OPS = "MID"
# HaplotypeCaller's haplotype-to-reference parameters (GATK 3.6, [EXT], reading R20)
GATK_HC = (200, -150, -260, -11)


class Params(ctypes.Structure):
    _fields_ = [("match", ctypes.c_int32), ("mismatch", ctypes.c_int32), ("open", ctypes.c_int32),
                ("extend", ctypes.c_int32)]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            vp = ctypes.c_void_p
            L.sw_align.argtypes = [ctypes.c_int64, ctypes.c_int64, vp, vp, ctypes.POINTER(Params), ctypes.c_int,
                                   vp, vp, vp, vp]
            L.sw_align.restype = ctypes.c_int64
            L.sw_batch.argtypes = [vp, vp, vp, vp, vp, ctypes.c_int64, ctypes.POINTER(Params), vp, vp, vp,
                                   ctypes.c_int]
            L.sw_batch.restype = ctypes.c_int
            _lib = L
    return _lib


def _u8(x) -> np.ndarray:
    if isinstance(x, (bytes, bytearray)):
        return np.frombuffer(bytes(x), dtype=np.uint8).copy()
    if isinstance(x, str):
        return np.frombuffer(x.encode("ascii"), dtype=np.uint8).copy()
    return np.ascontiguousarray(np.asarray(x, dtype=np.uint8))


def cigar_string(ops) -> str:
    return "".join(f"{int(o) >> 4}{OPS[int(o) & 15]}" for o in ops)


def align(a, b, params=GATK_HC, literal: bool = False) -> dict:
    """One alignment of a (rows) against b (columns). Returns H, btrack ((M+1) x (N+1)),
    score, end (i, j), start (i, j), ops and the CIGAR string."""
    a, b = _u8(a), _u8(b)
    M, N = a.size, b.size
    H = np.zeros((M + 1, N + 1), dtype=np.int32)
    bt = np.zeros((M + 1, N + 1), dtype=np.int32)
    res = np.zeros(5, dtype=np.int32)
    ops = np.zeros(M + N + 1, dtype=np.uint32)
    p = Params(*params)
    n = lib().sw_align(M, N, a.ctypes.data, b.ctypes.data, ctypes.byref(p), int(literal), H.ctypes.data,
                       bt.ctypes.data, res.ctypes.data, ops.ctypes.data)
    ops = ops[:n].copy()
    return {"H": H, "bt": bt, "score": int(res[0]), "end": (int(res[1]), int(res[2])),
            "start": (int(res[3]), int(res[4])), "ops": ops, "cigar": cigar_string(ops)}


def ops_offsets(ref_offsets, alt_offsets, tasks) -> np.ndarray:
    """Per-task offset of its CIGAR runs in the ops buffer: prefix sum of M_t + N_t."""
    ro, ao, t = np.asarray(ref_offsets), np.asarray(alt_offsets), np.asarray(tasks).reshape(-1, 2)
    cap = (ro[t[:, 0] + 1] - ro[t[:, 0]]) + (ao[t[:, 1] + 1] - ao[t[:, 1]])
    return np.concatenate([[0], np.cumsum(cap)]).astype(np.int64)


def batch(ref, ref_offsets, alt, alt_offsets, tasks, params=GATK_HC, nthreads: int = 0):
    """All tasks (ref_idx, alt_idx). Returns (res n x 6 [score, end_i, end_j, start_i,
    start_j, n_ops], ops, ops_off)."""
    ref, alt = _u8(ref), _u8(alt)
    ro = np.ascontiguousarray(ref_offsets, dtype=np.int64)
    ao = np.ascontiguousarray(alt_offsets, dtype=np.int64)
    t = np.ascontiguousarray(np.asarray(tasks, dtype=np.int32).reshape(-1, 2))
    n = t.shape[0]
    off = ops_offsets(ro, ao, t)
    res = np.zeros((n, 6), dtype=np.int32)
    ops = np.zeros(max(int(off[-1]), 1), dtype=np.uint32)
    p = Params(*params)
    nt = nthreads or (os.cpu_count() or 1)
    rc = lib().sw_batch(ref.ctypes.data, ro.ctypes.data, alt.ctypes.data, ao.ctypes.data, t.ctypes.data, n,
                        ctypes.byref(p), res.ctypes.data, ops.ctypes.data, off.ctypes.data, nt)
    if rc != 0:
        raise MemoryError("sw_batch failed")
    return res, ops, off


def rescore(a, b, start, ops, params=GATK_HC) -> int:
    """Score of the alignment a CIGAR describes (Eq. 5's terms along the path): an
    independent check of a traceback."""
    a, b = _u8(a), _u8(b)
    match, mismatch, op_, ext = params
    i, j = start[0] - 1, start[1] - 1
    s = 0
    for o in ops:
        ln, op = int(o) >> 4, int(o) & 15
        if op == 0:
            for _ in range(ln):
                s += match if a[i] == b[j] else mismatch
                i += 1
                j += 1
        elif op == 1:
            s += op_ + (ln - 1) * ext
            j += ln
        else:
            s += op_ + (ln - 1) * ext
            i += ln
    return s, (i, j)
