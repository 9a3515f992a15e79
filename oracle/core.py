"""ctypes binding of the plain-C PairHMM oracle (oracle/phmm_oracle.c).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py). Shares no code with the
CUDA product path. The C file's header states what is computed and cites
PAPER.md (Eq. 6 at L18@541, termination at L20@2262) for every step.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "phmm_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_u8p = ctypes.POINTER(ctypes.c_uint8)
_i64p = ctypes.POINTER(ctypes.c_int64)
_i32p = ctypes.POINTER(ctypes.c_int32)
_f64p = ctypes.POINTER(ctypes.c_double)


def build(force: bool = False) -> str:
    """Compile phmm_oracle.c with plain -O2 (no intrinsics, no -ffast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-o", tmp, _SRC, "-lm"]
        )
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            L.oracle_prob_parts.argtypes = [ctypes.c_int64, ctypes.c_int64] + [_f64p] * 8 + [_f64p] * 3
            L.oracle_prob_parts.restype = ctypes.c_int
            L.oracle_phred_parts.argtypes = [_u8p] * 5 + [ctypes.c_int64, _u8p, ctypes.c_int64] + [_f64p] * 3
            L.oracle_phred_parts.restype = ctypes.c_int
            L.oracle_batch.argtypes = [_u8p] * 5 + [_i64p, ctypes.c_int64, _u8p, _i64p, ctypes.c_int64,
                                                    _i32p, ctypes.c_int64, _f64p, ctypes.c_int]
            L.oracle_batch.restype = ctypes.c_int
            L.oracle_max_threads.argtypes = []
            L.oracle_max_threads.restype = ctypes.c_int
            _lib = L
    return _lib


def _p(a: np.ndarray, t):
    return a.ctypes.data_as(t)


def _u8(x) -> np.ndarray:
    if isinstance(x, (bytes, bytearray)):
        return np.frombuffer(bytes(x), dtype=np.uint8).copy()
    if isinstance(x, str):
        return np.frombuffer(x.encode("ascii"), dtype=np.uint8).copy()
    return np.ascontiguousarray(np.asarray(x, dtype=np.uint8))


def prob_parts(alpha, beta, gamma, delta, eps, zeta, mu, prior):
    """Probability-domain core. Per-row transition arrays (length m, destination
    row i at index i-1) and an (m, N) emission matrix. Returns
    (log10 sum M(m,.), log10 sum I(m,.), log10 P)."""
    prior = np.ascontiguousarray(np.asarray(prior, dtype=np.float64))
    m, n = prior.shape
    arrs = [np.ascontiguousarray(np.asarray(a, dtype=np.float64).reshape(m)) for a in
            (alpha, beta, gamma, delta, eps, zeta, mu)]
    out = np.zeros(3, dtype=np.float64)
    rc = lib().oracle_prob_parts(m, n, *[_p(a, _f64p) for a in arrs], _p(prior, _f64p),
                                 _p(out[0:1], _f64p), _p(out[1:2], _f64p), _p(out[2:3], _f64p))
    if rc != 0:
        raise ValueError("oracle_prob_parts failed")
    return float(out[0]), float(out[1]), float(out[2])


def phred_parts(read, q, qi, qd, qg, hap):
    """Phred wrapper for one pair: returns (log10 M-part, log10 I-part, log10 P)."""
    r, q, qi, qd, qg, h = (_u8(x) for x in (read, q, qi, qd, qg, hap))
    m, n = r.size, h.size
    if not (q.size == qi.size == qd.size == qg.size == m):
        raise ValueError("quality arrays must match the read length")
    out = np.zeros(3, dtype=np.float64)
    rc = lib().oracle_phred_parts(_p(r, _u8p), _p(q, _u8p), _p(qi, _u8p), _p(qd, _u8p), _p(qg, _u8p),
                                  m, _p(h, _u8p), n,
                                  _p(out[0:1], _f64p), _p(out[1:2], _f64p), _p(out[2:3], _f64p))
    if rc != 0:
        raise ValueError("oracle_phred_parts failed")
    return float(out[0]), float(out[1]), float(out[2])


def phred_log10(read, q, qi, qd, qg, hap) -> float:
    return phred_parts(read, q, qi, qd, qg, hap)[2]


def batch_log10(batch, pair_idx=None, nthreads: int = 0) -> np.ndarray:
    """log10 P for every pair of a batch (the library's layout: concatenated
    bytes + int64 offsets + int32 (read, hap) pairs). ``pair_idx`` restricts
    the computation to a subset of pairs (returned in that order)."""
    pairs = np.ascontiguousarray(batch.pairs, dtype=np.int32).reshape(-1, 2)
    if pair_idx is not None:
        pairs = np.ascontiguousarray(pairs[np.asarray(pair_idx)])
    n_pairs = pairs.shape[0]
    out = np.full(n_pairs, np.nan, dtype=np.float64)
    arrs = [np.ascontiguousarray(a, dtype=np.uint8) for a in
            (batch.read_bases, batch.base_quals, batch.ins_quals, batch.del_quals, batch.gcp_quals)]
    ro = np.ascontiguousarray(batch.read_offsets, dtype=np.int64)
    hb = np.ascontiguousarray(batch.hap_bases, dtype=np.uint8)
    ho = np.ascontiguousarray(batch.hap_offsets, dtype=np.int64)
    rc = lib().oracle_batch(*[_p(a, _u8p) for a in arrs], _p(ro, _i64p), ro.size - 1,
                            _p(hb, _u8p), _p(ho, _i64p), ho.size - 1,
                            _p(pairs, _i32p), n_pairs, _p(out, _f64p), int(nthreads))
    if rc != 0:
        raise IndexError("oracle_batch: pair index out of range")
    return out


def max_threads() -> int:
    return int(lib().oracle_max_threads())
