"""CPU-side checks of the C-ABI boundary: the library builds, loads and exports
every entry point include/phmm.h declares; the binding marshals the layout.
No compute call is made here (there is no GPU on the build box)."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_ipps_wangxc17_b200 import build, phmm, synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "phmm.h")


def _declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(phmm_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    build.build()
    return phmm.load_library()


def test_header_declares_the_north_star_entry_points():
    decl = _declared_functions()
    for name in ("phmm_create", "phmm_compute_batch", "phmm_destroy"):
        assert name in decl


def test_library_exports_every_declared_symbol(lib):
    for name in _declared_functions():
        assert hasattr(lib, name), name
    assert sorted(phmm.EXPORTED_SYMBOLS) == _declared_functions()


def test_abi_version_and_status_strings(lib):
    import re

    hdr = open(os.path.join(ROOT, "include", "phmm.h")).read()
    assert lib.phmm_abi_version() == int(re.search(r"#define PHMM_ABI_VERSION (\d+)", hdr).group(1))
    for code in (0, -1, -2, -3, -4, -5, -6, -7):
        s = lib.phmm_status_string(code).decode()
        assert s and s != "unknown status"
    assert lib.phmm_status_string(-99).decode() == "unknown status"


def test_null_safety_without_gpu(lib):
    # destroy(NULL) is a no-op; create(NULL) is an argument error
    lib.phmm_destroy(None)
    assert lib.phmm_create(None, None) == -1
    st = phmm._Stats()
    assert lib.phmm_get_stats(None, ctypes.byref(st)) == -1
    assert lib.phmm_compute_batch(None, None, None, None) == -1


def test_create_without_gpu_reports_cuda_error(lib):
    import torch

    if torch.cuda.is_available():
        pytest.skip("GPU present")
    h = ctypes.c_void_p()
    cfg = phmm._Config()
    rc = lib.phmm_create(ctypes.byref(h), ctypes.byref(cfg))
    assert rc in (-6, -1)
    assert not h.value


def test_host_struct_marshals_layout():
    b = synth.random_pairs_batch(1, 7)
    s, keep = phmm._host_struct(b)
    assert s.n_pairs == 7 and s.n_reads == 7 and s.n_haps == 7
    assert s.total_read_bases == int(b.read_offsets[-1])
    assert s.total_hap_bases == int(b.hap_offsets[-1])
    assert s.read_bases == keep["read_bases"].ctypes.data
    assert keep["pairs"].dtype == np.int32 and keep["pairs"].size == 14


def test_product_path_does_not_import_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_wangxc17_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f), errors="ignore").read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "phmm_oracle" not in txt and "liboracle" not in txt, f


def test_sw_entry_points_reject_null_without_gpu(lib):
    """The Smith-Waterman calls validate their arguments before touching the device."""
    assert lib.phmm_sw_align_batch(None, None, None, None, None) == -1
    assert lib.phmm_sw_align_batch_dev(None, None, None, None, None) == -1


def test_device_batch_checks_dtypes_and_sizes_on_cpu_tensors():
    """DeviceBatch.check (the binding's marshalling guard) on CPU tensors: wrong dtype,
    non-contiguous or mismatched sizes raise ValueError before any library call."""
    import torch

    b = synth.random_pairs_batch(1, 5)
    db = phmm.DeviceBatch.from_host(b, device="cpu")
    db.check()
    bad = phmm.DeviceBatch(**{**db.__dict__, "pairs": db.pairs.to(torch.int64)})
    with pytest.raises(ValueError):
        bad.check()
    bad = phmm.DeviceBatch(**{**db.__dict__, "ins_quals": db.ins_quals[:-1]})
    with pytest.raises(ValueError):
        bad.check()
    bad = phmm.DeviceBatch(**{**db.__dict__, "read_offsets": db.read_offsets.repeat(2)[::2]})
    with pytest.raises(ValueError):
        bad.check()
    with pytest.raises(ValueError):
        phmm._check_out(torch.empty(3, dtype=torch.float32), torch.float64, 3, torch.device("cpu"), "out")


def test_submit_and_wait_reject_null_without_gpu(lib):
    t = ctypes.c_uint64()
    assert lib.phmm_submit(None, None, None, None, ctypes.byref(t)) == -1
    assert lib.phmm_wait(None, 1) == -1
