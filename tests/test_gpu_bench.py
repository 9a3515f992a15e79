"""bench.py on the GPU keeps the driver's JSON contract (one line; value, roofline, e2e,
clocks, gpu_launches, cpu_baseline) on a reduced C2 shard."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--regions", "512", "--steps", "3",
                        "--warmup", "3", "--cpu-seconds", "1"], capture_output=True, text=True, timeout=900,
                       cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "gpu_launches", "roofline", "cpu_baseline", "e2e", "clocks"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["warmup"] == 3 and d["value"] > 0
    assert d["gpu_launches"] > 0 and d["scaling"] == "weak" and d["vs_baseline"] is None
    rf = d["roofline"]
    assert rf["bound"] == "alu" and 0 < rf["frac"] < 1 and rf["achieved"] > d["value"]
    e = d["e2e"]
    assert 0 < e["value"] <= d["value"] * 1.05 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert 0 < e["pageable"]["value"] <= d["value"] * 1.05
    assert len(d["result_sha256"]) == 64
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["cores"] >= 1 and c["parity_max_abs_log10"] <= 1e-3
    assert d["clocks"]["samples"] >= 1


def test_bench_c5_strong_split_line():
    """--workload C5 (strong split of a fixed region set; here 64 regions = 16,384 pairs at
    N = 1): the job's pairs and cells, and the result hash of the job in global pair order."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--workload", "C5", "--regions", "64",
                        "--steps", "3", "--warmup", "3", "--no-e2e", "--no-cpu-baseline"], capture_output=True,
                       text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.strip()][-1])
    assert d["scaling"] == "strong" and d["config"]["job_pairs"] == 64 * 32 * 8
    assert d["config"]["job_cells"] == d["config"]["cells_rank0"]
    from paper_conf_ipps_wangxc17_b200 import synth
    assert d["config"]["job_cells"] == synth.config_batch("C5", n_regions=64).cells()
    assert len(d["result_sha256"]) == 64


def _free_port():
    import socket

    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _bench_line(args, nproc=1, env_extra=None):
    env = dict(os.environ, **(env_extra or {}))
    if nproc == 1:
        cmd = [sys.executable, os.path.join(ROOT, "bench.py")] + args
    else:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
               "--master-addr", "127.0.0.1", f"--master-port={_free_port()}", os.path.join(ROOT, "bench.py"),
               "--gpus", str(nproc)] + args
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1200, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_multi_rank_path_is_bitwise_across_rank_counts():
    """bench.py's N > 1 path end to end on the one GPU of the test box (ranks share it; the
    result gather goes through gloo and host memory, PHMM_BENCH_BACKEND=gloo): the strong
    split of a fixed C5 region set gives the same job results (result_sha256) at N = 1, 2 and 4,
    with every rank's shard, the slot all-gather and the global reorder of parallel.py; the
    weak split reports every rank's cells."""
    args = ["--workload", "C5", "--regions", "24", "--steps", "2", "--warmup", "3", "--no-cpu-baseline"]
    one = _bench_line(args)
    for n in (2, 4):
        d = _bench_line(args, nproc=n, env_extra={"PHMM_BENCH_BACKEND": "gloo"})
        assert d["n_gpus"] == n and d["scaling"] == "strong"
        assert d["config"]["job_cells"] == one["config"]["job_cells"]
        assert d["result_sha256"] == one["result_sha256"], n
        assert d["e2e"]["value"] > 0 and d["e2e"]["streamed"]["value"] > 0
    w = _bench_line(["--workload", "C2", "--regions", "8", "--steps", "2", "--warmup", "3", "--no-cpu-baseline",
                     "--no-e2e", "--no-extra"], nproc=2, env_extra={"PHMM_BENCH_BACKEND": "gloo"})
    assert w["scaling"] == "weak" and w["config"]["job_pairs"] == 2 * 8 * 16 * 8
