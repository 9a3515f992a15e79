"""The host-side helpers of the pipelined host call (csrc/host_stage.h), built with g++ and run
on the CPU: streaming-store memcpy at every alignment / length class, CopyPool::memcpy_par and
CopyPool::for_each (tests/cpp/host_stage_test.cpp). No GPU and no CUDA call."""
import os
import shutil
import subprocess

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
CUDA_INC = "/usr/local/cuda/include"


@pytest.mark.skipif(shutil.which("g++") is None or not os.path.isdir(CUDA_INC), reason="needs g++ and CUDA headers")
def test_host_stage_helpers(tmp_path):
    exe = tmp_path / "host_stage_test"
    r = subprocess.run(["g++", "-O2", "-std=c++17", "-pthread", f"-I{CUDA_INC}", os.path.join(HERE, "cpp", "host_stage_test.cpp"),
                        "-o", str(exe)], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr[-3000:]
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0 and r.stdout.strip() == "ok", r.stdout + r.stderr
