"""The paper's microbenchmark methodology (Eq. 1-4) and performance model (Eq. 7-8),
re-run on sm_100a (paper_conf_ipps_wangxc17_b200/shuffle_study.py).

CPU tests pin the host arithmetic against hand-computed values; GPU tests run the
Listing 1 kernels and the design-A (shared-memory exchange) build of the wavefront
kernel against the oracle.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

from paper_conf_ipps_wangxc17_b200 import shuffle_study as ss

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_fit_line_exact_and_noisy():
    it = np.arange(1000, 11000, 1000)
    k, beta, r2 = ss.fit_line(it, 7.0 * it + 250.0)
    assert k == pytest.approx(7.0, abs=1e-9) and beta == pytest.approx(250.0, abs=1e-6) and r2 == pytest.approx(1.0)
    rng = np.random.default_rng(0)
    k2, _, r22 = ss.fit_line(it, 31.0 * it + 90.0 + rng.normal(0, 20.0, it.size))
    assert abs(k2 - 31.0) < 0.05 and r22 > 0.999
    with pytest.raises(ValueError):
        ss.fit_line([5, 5], [1, 2])


def test_eq1_to_eq4_recover_known_latencies():
    """Build slopes from known latencies with the paper's model t = it*(lat + alpha) + beta:
    k_reg = 1 + alpha, k_shfl = lat_shfl + alpha, k_smem = lat_smem + alpha,
    k_sync = lat_smem + lat_sync + alpha (the sync kernel also chases a pointer)."""
    alpha, lat = 4.0, {"shfl_up_1": 26.0, "shfl_idx_random": 27.5, "sharedmem": 29.0}
    lat_sync = 57.0
    slopes = {"reg": 1.0 + alpha}
    slopes.update({n: v + alpha for n, v in lat.items()})
    slopes["sharedmemsync_32"] = lat["sharedmem"] + lat_sync + alpha
    got = ss.derive_latencies(slopes)
    assert got["reg"] == 1.0
    for n, v in lat.items():
        assert got[n] == pytest.approx(v)
    assert got["sharedmemsync_32"] == pytest.approx(lat_sync)


def test_eq4_is_eq3_minus_the_shared_access():
    assert ss.sync_latency(k_sync=100.0, k_reg=5.0, latency_sharedmem=29.0) == pytest.approx(1 + 100 - 5 - 29)
    assert ss.latency_from_slopes(33.0, 5.0) == pytest.approx(29.0)


def test_eq7_parallelism_hand_values():
    p = ss.Platform(n_sm=148, regs_per_sm=65536, smem_per_sm=233472, threads_per_sm=2048, freq_hz=1.965e9)
    k = ss.KernelChar("wf", regs_per_thread=234, smem_per_block=81920, threads_per_block=128)
    # min(65536/234, 233472/81920*128) = min(280.068..., 364.8) -> 148 * 280.068...
    assert ss.parallelism_eq7(p, k) == pytest.approx(148 * 65536 / 234)
    # resident: 234 regs -> 7488/warp -> 7680 (units of 256) -> 2 blocks of 4 warps; smem 2 blocks
    assert ss.parallelism_resident(p, k) == 148 * 2 * 128
    # smem-bound case: 100 KB blocks -> 2 per SM (with 1 KB reserved each)
    k2 = ss.KernelChar("smem", regs_per_thread=32, smem_per_block=100 * 1024, threads_per_block=128)
    assert ss.parallelism_resident(p, k2) == 148 * 2 * 128
    assert ss.parallelism_eq7(p, k2) == pytest.approx(148 * 233472 / (100 * 1024) * 128)


def test_eq8_and_inverse():
    perf = ss.performance_eq8(parallelism=37888, freq_hz=1.965e9, latency_cycles=456.0, cells_per_thread_iter=16)
    assert perf == pytest.approx(37888 * 16 * 1.965e9 / 456.0)
    assert ss.implied_latency(perf, 37888, 1.965e9, 16) == pytest.approx(456.0)
    # the paper's single-cell form
    assert ss.performance_eq8(1000, 1e9, 10.0) == pytest.approx(1e11)


def test_throughput_aware_latency_takes_the_binding_term():
    c = ss.StepCost(instructions=102, fma_pipe_cycles=120, critical_path=90, warps_per_scheduler=2)
    assert ss.latency_throughput_aware(c) == 240
    c2 = ss.StepCost(instructions=10, fma_pipe_cycles=10, critical_path=90, warps_per_scheduler=2)
    assert ss.latency_throughput_aware(c2) == 90


def test_microbenchmark_plan_covers_listing1_and_fig1():
    names = [p[0] for p in ss.microbenchmark_plan()]
    assert "reg" in names and "sharedmem" in names
    assert any(n.startswith("sharedmemsync") for n in names)
    for v in ("shfl_idx", "shfl_up", "shfl_down", "shfl_xor"):
        assert any(n.startswith(v) for n in names)


@pytest.mark.gpu
def test_latency_microbenchmarks_on_gpu():
    # min of 3 repeats: a single cold first launch (instruction cache) can bend the line
    res = ss.run_microbenchmarks(iterations=(1000, 2000, 3000, 4000, 5000), repeats=3)
    lat = ss.latency_table(res)
    for r in res:
        assert r.r2 > 0.999, (r.name, r.r2)  # t is linear in #iterations (Eq. 1)
    assert 5 < lat["shfl_idx_random"] < 100
    assert 5 < lat["sharedmem"] < 100
    assert all(5 < lat[n] < 100 for n in lat if n.startswith("shfl"))


@pytest.mark.gpu
def test_design_a_library_parity():
    """libphmm_xsmem.so (row exchange through a shared-memory line buffer) computes the
    same results as the oracle (and bitwise the same as the shuffle build)."""
    lib = os.path.join(ROOT, "paper_conf_ipps_wangxc17_b200", "libphmm_xsmem.so")
    assert os.path.exists(lib), "build_all() builds the design-A library"
    code = r"""
import numpy as np, sys
sys.path.insert(0, %r)
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
b = synth.concat_batches([synth.config_batch("C1"), synth.config_batch("C2", n_regions=8),
                          synth.random_pairs_batch(5, 300, m_range=(1, 60), n_range=(1, 60))])
ref = oracle.batch_log10(b)
with phmm.PairHMM(precision="fp32") as h:
    got, _ = h.compute_batch(b)
fin = np.isfinite(ref)
assert np.array_equal(np.isneginf(got), np.isneginf(ref))
d = float(np.max(np.abs(got[fin] - ref[fin])))
assert d <= 1e-3, d
np.save(sys.argv[1], got)
print("ok", d)
""" % ROOT
    outs = []
    for libpath, tag in ((lib, "a"), (os.path.join(ROOT, "paper_conf_ipps_wangxc17_b200", "libphmm.so"), "b")):
        fn = f"/tmp/phmm_design_{tag}_{os.getpid()}.npy"
        r = subprocess.run([sys.executable, "-c", code, fn], env=dict(os.environ, PHMM_LIB=libpath),
                           capture_output=True, text=True, cwd=ROOT)
        assert r.returncode == 0, r.stderr[-3000:]
        outs.append(np.load(fn))
        os.unlink(fn)
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("lib", ["libphmm.so", "libphmm_xsmem.so"])
def test_hot_loop_mix_finds_the_wavefront_kernel(lib):
    """The study's SASS / ptxas lookups name the kernel that the libraries actually contain
    (a stale symbol would silently drop the design comparison's instruction mix)."""
    so = os.path.join(ROOT, "paper_conf_ipps_wangxc17_b200", lib)
    if not os.path.exists(so):
        pytest.skip("library not built")
    mix = ss.hot_loop_mix(so, ss.WF32_SYMBOL)
    # one group of 4 steps x 16 cells per lane: the 5-op rescaled cell is 320 FP32 lane-ops
    fp_ops = 2 * (mix.get("FFMA2", 0) + mix.get("FMUL2", 0) + mix.get("FADD2", 0)) + \
        mix.get("FFMA", 0) + mix.get("FMUL", 0) + mix.get("FADD", 0)
    assert fp_ops == 320, mix
    assert mix.get("SHFL", 0) > 0 if lib == "libphmm.so" else mix.get("STS", 0) > mix.get("SHFL", 0)
    ptx = os.path.join(ROOT, "paper_conf_ipps_wangxc17_b200",
                       "ptxas_info.txt" if lib == "libphmm.so" else lib + ".ptxas.txt")
    if os.path.exists(ptx):
        assert 0 < ss._ptxas_regs(ptx, ss.WF32_SYMBOL) <= 255
