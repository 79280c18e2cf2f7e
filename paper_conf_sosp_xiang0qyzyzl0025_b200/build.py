"""Build libaegkv.so (the product: C-ABI + runtime + sm_100a kernels) and libaeginputs.so (test/bench
input generator and checker kernels) in-tree, with nvcc for sm_100a.  Incremental by mtime.

    python -m paper_conf_sosp_xiang0qyzyzl0025_b200.build [--force]
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
LIB_DIR = os.path.join(PKG, "lib")
OBJ_DIR = os.path.join(ROOT, "build", "obj")

CXXFLAGS = ["-O2", "-g", "-fPIC", "-std=c++17", "-Wall", "-Wno-unused-function", "-pthread"]
NVFLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v"]
# experiments only (tools/*.sh): extra -D flags for the kernels, e.g. "-DAEG_BW_GRID=120"
NVFLAGS += os.environ.get("AEG_NVCC_EXTRA", "").split()
CXXFLAGS += os.environ.get("AEG_CXX_EXTRA", "").split()   # same, for the runtime (e.g. swap.cc)


def _needs(out: str, deps: list[str]) -> bool:
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd: list[str], log: list[str]):
    r = subprocess.run(cmd, capture_output=True, text=True)
    log.append(" ".join(cmd) + "\n" + r.stdout + r.stderr)
    if r.returncode != 0:
        raise RuntimeError(f"build failed:\n{' '.join(cmd)}\n{r.stdout}\n{r.stderr}")


def _build_lib(name: str, srcs: list[str], incs: list[str], headers: list[str], force: bool, log: list[str]) -> str:
    os.makedirs(OBJ_DIR, exist_ok=True)
    os.makedirs(LIB_DIR if name == "libaegkv.so" else os.path.dirname(srcs[0]), exist_ok=True)
    out = os.path.join(LIB_DIR, name) if name == "libaegkv.so" else os.path.join(ROOT, "aeg_inputs", name)
    objs, jobs = [], []
    inc = [f"-I{d}" for d in incs] + [f"-I{CUDA}/include"]
    for s in srcs:
        o = os.path.join(OBJ_DIR, name + "." + os.path.relpath(s, ROOT).replace(os.sep, "_") + ".o")
        objs.append(o)
        if force or _needs(o, [s] + headers):
            if s.endswith(".cu"):
                jobs.append([NVCC] + NVFLAGS + inc + ["-c", s, "-o", o])
            else:
                jobs.append(["g++"] + CXXFLAGS + inc + ["-c", s, "-o", o])
    with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        for f in [ex.submit(_run, j, log) for j in jobs]:
            f.result()
    if force or jobs or _needs(out, objs):
        tmp = out + ".tmp"
        _run([NVCC] + ARCH + ["-shared", "-cudart", "shared", "-Xlinker", f"-rpath,{CUDA}/lib64", "-o", tmp]
             + objs + ["-lpthread"], log)
        os.replace(tmp, out)
    return out


def build(force: bool = False, verbose: bool = False) -> list[str]:
    if not os.path.exists(NVCC) and shutil.which("nvcc") is None:
        raise RuntimeError("nvcc not found: the CUDA toolkit is required to build libaegkv.so")
    log: list[str] = []
    csrc = os.path.join(PKG, "csrc")
    inc = os.path.join(ROOT, "include")
    headers = glob.glob(os.path.join(csrc, "**", "*.h"), recursive=True) + [os.path.join(inc, "aeg.h")]
    srcs = sorted(glob.glob(os.path.join(csrc, "**", "*.cc"), recursive=True)
                  + glob.glob(os.path.join(csrc, "**", "*.cu"), recursive=True))
    outs = [_build_lib("libaegkv.so", srcs, [inc, csrc], headers, force, log)]
    isrc = os.path.join(ROOT, "aeg_inputs", "csrc")
    outs.append(_build_lib("libaeginputs.so", sorted(glob.glob(os.path.join(isrc, "*.cu"))), [isrc],
                           glob.glob(os.path.join(isrc, "*.h")), force, log))
    os.makedirs(os.path.join(ROOT, "build"), exist_ok=True)
    with open(os.path.join(ROOT, "build", "build.log"), "w") as f:
        f.write("\n".join(log))
    if verbose:
        print("\n".join(log))
    return outs


if __name__ == "__main__":
    print("\n".join(build(force="--force" in sys.argv, verbose="-v" in sys.argv)))
