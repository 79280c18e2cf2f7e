"""The boundary from plain C (examples/c_client.c): include/aeg.h + libaegkv.so, no Python binding,
no PyTorch.  CPU: the host-only allocator mode.  GPU: a Qwen-7B-shaped swap round trip with per-layer
readiness, every byte compared by the C program itself."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_sosp_xiang0qyzyzl0025_b200", "lib")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")


def _build(tmp_path):
    from paper_conf_sosp_xiang0qyzyzl0025_b200 import build
    build.build()
    exe = str(tmp_path / "c_client")
    subprocess.run(["gcc", "-O2", "-std=c11", "-Wall", "-I", os.path.join(ROOT, "include"), "-o", exe,
                    os.path.join(ROOT, "examples", "c_client.c"), "-L", LIB, "-laegkv",
                    "-L", os.path.join(CUDA, "lib64"), "-lcudart", f"-Wl,-rpath,{LIB}",
                    f"-Wl,-rpath,{os.path.join(CUDA, 'lib64')}"], check=True)
    return exe


def test_c_client_host_mode(tmp_path):
    exe = _build(tmp_path)
    r = subprocess.run([exe, "host"], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "allocator OK" in r.stdout


@pytest.mark.gpu
def test_c_client_gpu_round_trip(tmp_path):
    from .gpu_harness import require_gpu
    require_gpu()
    exe = _build(tmp_path)
    r = subprocess.run([exe, "gpu"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "every byte identical" in r.stdout
