"""Thin Python binding of libphmm (include/phmm.h) -- argument marshalling only.

Every step of the PairHMM path (validation, per-read tables, binning, the
wavefront, the FP64 rescue, log10) runs inside libphmm.so on the GPU. This
module never computes a likelihood itself and has no CPU fallback: if the
library cannot be loaded it raises.

Names follow the C ABI: ``phmm_create`` -> ``PairHMM(...)``,
``phmm_compute_batch`` -> ``PairHMM.compute_batch`` (host buffers),
``phmm_compute_batch_dev`` -> ``PairHMM.compute_batch_dev`` (torch CUDA
tensors), ``phmm_destroy`` -> ``PairHMM.close``.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PHMM_LIB") or os.path.join(_PKG, "libphmm.so")

PHMM_OK = 0
STATUS_NAMES = {
    0: "PHMM_OK", -1: "PHMM_E_INVALID_ARG", -2: "PHMM_E_INVALID_BASE", -3: "PHMM_E_INVALID_QUAL",
    -4: "PHMM_E_EMPTY_SEQ", -5: "PHMM_E_INDEX", -6: "PHMM_E_CUDA", -7: "PHMM_E_OOM",
}
PREC_FP64 = 0
PREC_FP32_RESCUE = 1
FLAG_TIMING = 1

_u8p = ctypes.POINTER(ctypes.c_uint8)
_i64p = ctypes.POINTER(ctypes.c_int64)
_i32p = ctypes.POINTER(ctypes.c_int32)
_f64p = ctypes.POINTER(ctypes.c_double)


class PhmmError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        super().__init__(f"{what}: {STATUS_NAMES.get(code, code)} ({status_string(code)})")


class _Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("precision", ctypes.c_int), ("cuda_stream", ctypes.c_void_p),
                ("flags", ctypes.c_uint32), ("col_bucket", ctypes.c_int32)]


class _Batch(ctypes.Structure):
    _fields_ = [("read_bases", ctypes.c_void_p), ("base_quals", ctypes.c_void_p),
                ("ins_quals", ctypes.c_void_p), ("del_quals", ctypes.c_void_p), ("gcp_quals", ctypes.c_void_p),
                ("read_offsets", ctypes.c_void_p), ("n_reads", ctypes.c_int64),
                ("hap_bases", ctypes.c_void_p), ("hap_offsets", ctypes.c_void_p), ("n_haps", ctypes.c_int64),
                ("pairs", ctypes.c_void_p), ("n_pairs", ctypes.c_int64),
                ("total_read_bases", ctypes.c_int64), ("total_hap_bases", ctypes.c_int64)]


class _Stats(ctypes.Structure):
    _fields_ = [("n_pairs", ctypes.c_int64), ("cells", ctypes.c_int64), ("padded_cells", ctypes.c_int64),
                ("n_rescued", ctypes.c_int64), ("n_fp64_underflow", ctypes.c_int64),
                ("n_chunks", ctypes.c_int32), ("kernel_launches", ctypes.c_int32),
                ("ms_total", ctypes.c_float), ("ms_h2d", ctypes.c_float), ("ms_prep", ctypes.c_float),
                ("ms_wavefront", ctypes.c_float), ("ms_rescue", ctypes.c_float),
                ("ms_finalize", ctypes.c_float), ("ms_d2h", ctypes.c_float), ("staged_bytes", ctypes.c_int64)]


class _SwBatch(ctypes.Structure):
    _fields_ = [("ref_bases", ctypes.c_void_p), ("ref_offsets", ctypes.c_void_p), ("n_refs", ctypes.c_int64),
                ("alt_bases", ctypes.c_void_p), ("alt_offsets", ctypes.c_void_p), ("n_alts", ctypes.c_int64),
                ("tasks", ctypes.c_void_p), ("n_tasks", ctypes.c_int64), ("total_ref_bases", ctypes.c_int64),
                ("total_alt_bases", ctypes.c_int64)]


class _SwParams(ctypes.Structure):
    _fields_ = [("match", ctypes.c_int32), ("mismatch", ctypes.c_int32), ("gap_open", ctypes.c_int32),
                ("gap_extend", ctypes.c_int32)]


# HaplotypeCaller's haplotype-to-reference Smith-Waterman parameters (R20)
SW_GATK_HC = (200, -150, -260, -11)
SW_OPS = "MID"

# every symbol include/phmm.h declares (checked by tests/test_abi.py)
EXPORTED_SYMBOLS = ("phmm_create", "phmm_compute_batch", "phmm_compute_batch_dev", "phmm_destroy",
                    "phmm_status_string", "phmm_get_stats", "phmm_abi_version", "phmm_set_stream", "phmm_submit", "phmm_wait",
                    "phmm_compute_batch_async", "phmm_sw_align_batch", "phmm_sw_align_batch_dev")

_lib = None


def load_library(path: str = LIB_PATH):
    """Load libphmm.so (raises if it is missing: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"libphmm.so not built ({path}); run `python -m paper_conf_ipps_wangxc17_b200.build` "
                           "or __graft_entry__.build()")
    L = ctypes.CDLL(path)
    L.phmm_create.argtypes = [ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(_Config)]
    L.phmm_create.restype = ctypes.c_int
    L.phmm_compute_batch.argtypes = [ctypes.c_void_p, ctypes.POINTER(_Batch), _f64p, _u8p]
    L.phmm_compute_batch.restype = ctypes.c_int
    L.phmm_compute_batch_dev.argtypes = [ctypes.c_void_p, ctypes.POINTER(_Batch), ctypes.c_void_p, ctypes.c_void_p]
    L.phmm_compute_batch_dev.restype = ctypes.c_int
    L.phmm_destroy.argtypes = [ctypes.c_void_p]
    L.phmm_destroy.restype = None
    L.phmm_status_string.argtypes = [ctypes.c_int]
    L.phmm_status_string.restype = ctypes.c_char_p
    L.phmm_get_stats.argtypes = [ctypes.c_void_p, ctypes.POINTER(_Stats)]
    L.phmm_get_stats.restype = ctypes.c_int
    L.phmm_abi_version.argtypes = []
    L.phmm_abi_version.restype = ctypes.c_int
    L.phmm_set_stream.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    L.phmm_set_stream.restype = ctypes.c_int
    L.phmm_submit.argtypes = [ctypes.c_void_p, ctypes.POINTER(_Batch), _f64p, _u8p, ctypes.POINTER(ctypes.c_uint64)]
    L.phmm_submit.restype = ctypes.c_int
    L.phmm_wait.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
    L.phmm_wait.restype = ctypes.c_int
    L.phmm_compute_batch_async.argtypes = [ctypes.c_void_p, ctypes.POINTER(_Batch), _f64p, _u8p,
                                           ctypes.POINTER(ctypes.c_uint64)]
    L.phmm_compute_batch_async.restype = ctypes.c_int
    for f in (L.phmm_sw_align_batch, L.phmm_sw_align_batch_dev):
        f.argtypes = [ctypes.c_void_p, ctypes.POINTER(_SwBatch), ctypes.POINTER(_SwParams), ctypes.c_void_p,
                      ctypes.c_void_p]
        f.restype = ctypes.c_int
    _lib = L
    return L


def status_string(code: int) -> str:
    try:
        return load_library().phmm_status_string(int(code)).decode()
    except Exception:  # noqa: BLE001 - only used for messages
        return "?"


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data if a.size else 0


def _host_struct(b) -> tuple:
    """(struct, keepalive) for a host batch (synth.Batch-like, numpy arrays)."""
    arrs = dict(
        read_bases=np.ascontiguousarray(b.read_bases, dtype=np.uint8),
        base_quals=np.ascontiguousarray(b.base_quals, dtype=np.uint8),
        ins_quals=np.ascontiguousarray(b.ins_quals, dtype=np.uint8),
        del_quals=np.ascontiguousarray(b.del_quals, dtype=np.uint8),
        gcp_quals=np.ascontiguousarray(b.gcp_quals, dtype=np.uint8),
        read_offsets=np.ascontiguousarray(b.read_offsets, dtype=np.int64),
        hap_bases=np.ascontiguousarray(b.hap_bases, dtype=np.uint8),
        hap_offsets=np.ascontiguousarray(b.hap_offsets, dtype=np.int64),
        pairs=np.ascontiguousarray(b.pairs, dtype=np.int32).reshape(-1),
    )
    s = _Batch()
    for k, v in arrs.items():
        setattr(s, k, _ptr(v))
    s.n_reads = arrs["read_offsets"].size - 1
    s.n_haps = arrs["hap_offsets"].size - 1
    s.n_pairs = arrs["pairs"].size // 2
    s.total_read_bases = int(arrs["read_offsets"][-1]) if arrs["read_offsets"].size else 0
    s.total_hap_bases = int(arrs["hap_offsets"][-1]) if arrs["hap_offsets"].size else 0
    return s, arrs


@dataclass
class DeviceBatch:
    """A batch resident on one CUDA device (torch tensors; torch is plumbing)."""

    read_bases: "object"
    base_quals: "object"
    ins_quals: "object"
    del_quals: "object"
    gcp_quals: "object"
    read_offsets: "object"
    hap_bases: "object"
    hap_offsets: "object"
    pairs: "object"  # int32 (n_pairs, 2)
    total_read_bases: int
    total_hap_bases: int

    @property
    def n_pairs(self) -> int:
        return int(self.pairs.shape[0])

    @staticmethod
    def from_host(b, device="cuda", pinned: bool = False, non_blocking: bool = False) -> "DeviceBatch":
        import torch

        def t(a, dt):
            x = torch.from_numpy(np.ascontiguousarray(a, dtype=dt))
            if pinned:
                x = x.pin_memory()
            return x.to(device, non_blocking=non_blocking)

        return DeviceBatch(read_bases=t(b.read_bases, np.uint8), base_quals=t(b.base_quals, np.uint8),
                           ins_quals=t(b.ins_quals, np.uint8), del_quals=t(b.del_quals, np.uint8),
                           gcp_quals=t(b.gcp_quals, np.uint8), read_offsets=t(b.read_offsets, np.int64),
                           hap_bases=t(b.hap_bases, np.uint8), hap_offsets=t(b.hap_offsets, np.int64),
                           pairs=t(np.asarray(b.pairs, dtype=np.int32).reshape(-1, 2), np.int32),
                           total_read_bases=int(b.read_offsets[-1]), total_hap_bases=int(b.hap_offsets[-1]))

    _DTYPES = dict(read_bases="uint8", base_quals="uint8", ins_quals="uint8", del_quals="uint8",
                   gcp_quals="uint8", read_offsets="int64", hap_bases="uint8", hap_offsets="int64", pairs="int32")

    def check(self) -> None:
        """Every tensor contiguous, of its ABI dtype and on the pairs' device; sizes
        consistent (the library validates the contents)."""
        dev = self.pairs.device
        for k, dt in self._DTYPES.items():
            x = getattr(self, k)
            if str(x.dtype) != "torch." + dt or not x.is_contiguous() or x.device != dev:
                raise ValueError(f"DeviceBatch.{k}: need a contiguous {dt} tensor on {dev}, got "
                                 f"{x.dtype} on {x.device} (contiguous={x.is_contiguous()})")
        if self.pairs.dim() != 2 or self.pairs.shape[1] != 2:
            raise ValueError("DeviceBatch.pairs must be (n_pairs, 2)")
        nr = int(self.read_bases.numel())
        for k in ("base_quals", "ins_quals", "del_quals", "gcp_quals"):
            if int(getattr(self, k).numel()) != nr:
                raise ValueError(f"DeviceBatch.{k} must have as many bytes as read_bases")
        if nr != int(self.total_read_bases) or int(self.hap_bases.numel()) != int(self.total_hap_bases):
            raise ValueError("DeviceBatch.total_read_bases / total_hap_bases disagree with the tensors")

    def struct(self) -> _Batch:
        s = _Batch()
        for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets",
                  "hap_bases", "hap_offsets", "pairs"):
            x = getattr(self, k)
            setattr(s, k, x.data_ptr() if x.numel() else 0)
        s.n_reads = int(self.read_offsets.numel()) - 1
        s.n_haps = int(self.hap_offsets.numel()) - 1
        s.n_pairs = int(self.pairs.shape[0])
        s.total_read_bases = int(self.total_read_bases)
        s.total_hap_bases = int(self.total_hap_bases)
        return s


def _check_out(t, dtype, n: int, dev, name: str) -> None:
    if t.dtype != dtype or not t.is_contiguous() or t.device != dev or t.numel() < n:
        raise ValueError(f"{name}: need a contiguous {dtype} tensor of >= {n} elements on {dev}, got "
                         f"{t.dtype}, {t.numel()} elements on {t.device} (contiguous={t.is_contiguous()})")


class Ticket:
    """A submitted batch (``phmm_submit`` / ``phmm_compute_batch_async``); ``wait()`` blocks in
    ``phmm_wait``. For a no-copy batch the ticket also keeps the input arrays alive."""

    def __init__(self, ctx, ticket: int, out, status, keep=None):
        self.ctx, self.ticket, self.out, self.status, self._keep = ctx, ticket, out, status, keep

    def wait(self):
        rc = self.ctx._L.phmm_wait(self.ctx._h, self.ticket)
        self._keep = None
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_wait")
        return self.out, self.status


class PairHMM:
    """One libphmm context (``phmm_create``) bound to one CUDA device."""

    def __init__(self, device: int = 0, precision: str = "fp32", stream=None, timing: bool = False,
                 col_bucket: int = 0):
        L = load_library()
        cfg = _Config()
        cfg.device = int(device)
        cfg.precision = {"fp64": PREC_FP64, "fp32": PREC_FP32_RESCUE, "fp32_rescue": PREC_FP32_RESCUE}[precision]
        cfg.cuda_stream = int(stream) if stream is not None else None
        cfg.flags = FLAG_TIMING if timing else 0
        cfg.col_bucket = int(col_bucket)
        h = ctypes.c_void_p()
        rc = L.phmm_create(ctypes.byref(h), ctypes.byref(cfg))
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_create")
        self._h = h
        self._L = L
        self.device = int(device)
        self.precision = precision
        # without an explicit stream the device variant follows torch's current stream
        # (set before every call), so it is ordered after the ops that produced its inputs
        self._follow_torch = stream is None
        self._cur_stream = None

    # ------------------------------------------------------------ host API
    def compute_batch(self, batch, out: Optional[np.ndarray] = None, status: Optional[np.ndarray] = None,
                      want_status: bool = True):
        """``phmm_compute_batch``: host buffers in, host log10 likelihoods out.
        ``out``/``status`` may be pre-allocated (e.g. pinned) numpy arrays."""
        s, keep = _host_struct(batch)
        n = int(s.n_pairs)
        if out is None:
            out = np.empty(n, dtype=np.float64)
        if status is None and want_status:
            status = np.empty(n, dtype=np.uint8)
        rc = self._L.phmm_compute_batch(self._h, ctypes.byref(s), out.ctypes.data_as(_f64p),
                                        status.ctypes.data_as(_u8p) if status is not None else None)
        del keep
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_compute_batch")
        return out, status

    def compute_batch_async(self, batch, out: Optional[np.ndarray] = None, status: Optional[np.ndarray] = None,
                            want_status: bool = True) -> "Ticket":
        """``phmm_compute_batch_async``: enqueue a host batch WITHOUT copying it (the ticket keeps
        the arrays alive; do not modify them before ``wait()``); the next submitted batch's inputs
        are copied to the device while this one computes when they are page-locked."""
        s, keep = _host_struct(batch)
        n = int(s.n_pairs)
        if out is None:
            out = np.empty(n, dtype=np.float64)
        if status is None and want_status:
            status = np.empty(n, dtype=np.uint8)
        t = ctypes.c_uint64()
        rc = self._L.phmm_compute_batch_async(self._h, ctypes.byref(s), out.ctypes.data_as(_f64p),
                                              status.ctypes.data_as(_u8p) if status is not None else None,
                                              ctypes.byref(t))
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_compute_batch_async")
        return Ticket(self, int(t.value), out, status, keep=(keep, s))

    def compute_batch_async_raw(self, s: _Batch, out_ptr: int, status_ptr: int = 0) -> int:
        """Direct ``phmm_compute_batch_async`` with prepared pointers (bench e2e leg); returns the
        ticket (raises on a submission error)."""
        t = ctypes.c_uint64()
        rc = int(self._L.phmm_compute_batch_async(self._h, ctypes.byref(s), ctypes.cast(out_ptr, _f64p),
                                                  ctypes.cast(status_ptr, _u8p) if status_ptr else None,
                                                  ctypes.byref(t)))
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_compute_batch_async")
        return int(t.value)

    def wait_raw(self, ticket: int) -> int:
        return int(self._L.phmm_wait(self._h, ctypes.c_uint64(ticket)))

    def compute_batch_raw(self, s: _Batch, out_ptr: int, status_ptr: int = 0) -> int:
        """Direct ``phmm_compute_batch`` with prepared pointers (bench e2e leg)."""
        return int(self._L.phmm_compute_batch(self._h, ctypes.byref(s), ctypes.cast(out_ptr, _f64p),
                                              ctypes.cast(status_ptr, _u8p) if status_ptr else None))

    # ------------------------------------------------------------ submission queue
    def submit(self, batch, out: Optional[np.ndarray] = None, status: Optional[np.ndarray] = None,
               want_status: bool = True) -> "Ticket":
        """``phmm_submit``: queue a host batch; returns a Ticket whose ``wait()`` (``phmm_wait``)
        returns (out, status) once the library has written them. The batch's inputs are
        copied by the call; ``out`` / ``status`` are kept alive by the ticket."""
        s, keep = _host_struct(batch)
        n = int(s.n_pairs)
        if out is None:
            out = np.empty(n, dtype=np.float64)
        if status is None and want_status:
            status = np.empty(n, dtype=np.uint8)
        t = ctypes.c_uint64()
        rc = self._L.phmm_submit(self._h, ctypes.byref(s), out.ctypes.data_as(_f64p),
                                 status.ctypes.data_as(_u8p) if status is not None else None, ctypes.byref(t))
        del keep
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_submit")
        return Ticket(self, int(t.value), out, status)

    # ------------------------------------------------------------ device API
    def set_stream(self, stream) -> None:
        """``phmm_set_stream``: enqueue later calls on ``stream`` (an int cudaStream_t,
        a torch.cuda.Stream, or None for the context's own stream)."""
        handle = getattr(stream, "cuda_stream", stream)
        rc = self._L.phmm_set_stream(self._h, int(handle) if handle else None)
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_set_stream")
        self._cur_stream = handle

    def compute_batch_dev(self, db: DeviceBatch, out=None, status=None, want_status: bool = True):
        """``phmm_compute_batch_dev``: torch CUDA tensors in and out. Unless the context was
        created on an explicit stream, the call runs on torch's current stream of the
        batch's device."""
        import torch

        n = db.n_pairs
        dev = db.pairs.device
        if dev.type != "cuda" or dev.index != self.device:
            raise ValueError(f"batch on {dev}, context on cuda:{self.device}")
        db.check()
        if out is None:
            out = torch.empty(n, dtype=torch.float64, device=dev)
        if status is None and want_status:
            status = torch.empty(n, dtype=torch.uint8, device=dev)
        _check_out(out, torch.float64, n, dev, "out")
        if status is not None:
            _check_out(status, torch.uint8, n, dev, "status")
        if self._follow_torch:
            cur = torch.cuda.current_stream(dev).cuda_stream
            if cur != self._cur_stream:
                self.set_stream(cur)
        s = db.struct()
        rc = self._L.phmm_compute_batch_dev(self._h, ctypes.byref(s), out.data_ptr() if n else None,
                                            status.data_ptr() if (status is not None and n) else None)
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_compute_batch_dev")
        return out, status

    # ------------------------------------------------------------ Smith-Waterman
    def sw_align_batch(self, b, params=SW_GATK_HC):
        """``phmm_sw_align_batch`` on a synth.SwBatch-like object (host numpy arrays).
        Returns (res int32 (n, 6): score, end_i, end_j, start_i, start_j, n_ops;
        ops uint32 CIGAR runs, all tasks back to back; ops_off int64 (n+1): where task
        t's runs start = prefix sums of n_ops)."""
        keep = [np.ascontiguousarray(b.ref_bases, dtype=np.uint8), np.ascontiguousarray(b.ref_offsets, dtype=np.int64),
                np.ascontiguousarray(b.alt_bases, dtype=np.uint8), np.ascontiguousarray(b.alt_offsets, dtype=np.int64),
                np.ascontiguousarray(np.asarray(b.tasks, dtype=np.int32).reshape(-1, 2))]
        rb, ro, ab, ao, t = keep
        n = t.shape[0]
        s = _SwBatch(rb.ctypes.data if rb.size else None, ro.ctypes.data, ro.size - 1,
                     ab.ctypes.data if ab.size else None, ao.ctypes.data, ao.size - 1,
                     t.ctypes.data if n else None, n, int(ro[-1]), int(ao[-1]))
        # output capacity sum(M + N) (indices clipped here; the library reports bad ones)
        ti, tj = np.clip(t[:, 0], 0, max(ro.size - 2, 0)), np.clip(t[:, 1], 0, max(ao.size - 2, 0))
        cap = (ro[ti + 1] - ro[ti]) + (ao[tj + 1] - ao[tj]) if n else np.zeros(0, np.int64)
        off = np.concatenate([[0], np.cumsum(cap)]).astype(np.int64)
        res = np.zeros((n, 6), dtype=np.int32)
        ops = np.zeros(max(int(off[-1]), 1), dtype=np.uint32)
        p = _SwParams(*params)
        rc = self._L.phmm_sw_align_batch(self._h, ctypes.byref(s), ctypes.byref(p), res.ctypes.data,
                                         ops.ctypes.data)
        del keep
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_sw_align_batch")
        packed = np.concatenate([[0], np.cumsum(res[:, 5].astype(np.int64))]).astype(np.int64)
        return res, ops[: max(int(packed[-1]), 0)], packed

    def sw_align_batch_dev(self, tensors: dict, params=SW_GATK_HC, res=None, ops=None):
        """``phmm_sw_align_batch_dev`` on torch CUDA tensors {ref_bases, ref_offsets,
        alt_bases, alt_offsets, tasks}; ``ops`` (int32 tensor) must hold sum(M + N)
        elements; the runs come back packed (task t's at the prefix sum of n_ops)."""
        import torch

        T = tensors
        n = int(T["tasks"].shape[0])
        s = _SwBatch(T["ref_bases"].data_ptr(), T["ref_offsets"].data_ptr(), T["ref_offsets"].numel() - 1,
                     T["alt_bases"].data_ptr(), T["alt_offsets"].data_ptr(), T["alt_offsets"].numel() - 1,
                     T["tasks"].data_ptr(), n, int(T["total_ref_bases"]), int(T["total_alt_bases"]))
        dev = T["tasks"].device
        if res is None:
            res = torch.empty((n, 6), dtype=torch.int32, device=dev)
        if self._follow_torch:
            cur = torch.cuda.current_stream(dev).cuda_stream
            if cur != self._cur_stream:
                self.set_stream(cur)
        p = _SwParams(*params)
        rc = self._L.phmm_sw_align_batch_dev(self._h, ctypes.byref(s), ctypes.byref(p), res.data_ptr(),
                                             ops.data_ptr())
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_sw_align_batch_dev")
        return res, ops

    def stats(self) -> dict:
        st = _Stats()
        rc = self._L.phmm_get_stats(self._h, ctypes.byref(st))
        if rc != PHMM_OK:
            raise PhmmError(rc, "phmm_get_stats")
        return {k: getattr(st, k) for k, _ in _Stats._fields_}

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._L.phmm_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass


def compute(batch, precision: str = "fp32", device: int = 0):
    """One-shot convenience: log10 P(read|hap) for every pair of a host batch."""
    with PairHMM(device=device, precision=precision) as h:
        return h.compute_batch(batch)
