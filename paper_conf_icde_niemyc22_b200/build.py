"""Build libtsplit.so in-tree: g++ for the host core, nvcc (sm_100a) for the
runtime and kernels, one shared library with a plain C ABI (include/ts.h).

    python -m paper_conf_icde_niemyc22_b200.build [--force]
"""

from __future__ import annotations

import glob
import hashlib
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libtsplit.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CXXFLAGS = ["-O2", "-std=c++17", "-fPIC", "-Wall", "-Wno-unused-function", f"-I{ROOT}/include"]
NVFLAGS = ARCH + ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", f"-I{ROOT}/include",
                  "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills"]


def sources():
    cpp = sorted(glob.glob(os.path.join(CSRC, "host", "*.cpp")))
    cu = sorted(glob.glob(os.path.join(CSRC, "runtime", "*.cu")) + glob.glob(os.path.join(CSRC, "kernels", "*.cu")))
    return cpp, cu


def _headers_digest():
    h = hashlib.sha1()
    for p in sorted(glob.glob(os.path.join(CSRC, "**", "*.h"), recursive=True) +
                    glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True) +
                    [os.path.join(ROOT, "include", "ts.h")]):
        h.update(open(p, "rb").read())
    return h.hexdigest()


def _obj(src, digest):
    h = hashlib.sha1(open(src, "rb").read() + digest.encode()).hexdigest()[:12]
    return os.path.join(BUILD, os.path.basename(src) + "." + h + ".o")


def _compile(src, digest):
    obj = _obj(src, digest)
    if os.path.exists(obj):
        return obj
    if src.endswith(".cu"):
        cmd = [NVCC] + NVFLAGS + ["-c", src, "-o", obj + ".tmp"]
    else:
        cmd = ["g++"] + CXXFLAGS + ["-c", src, "-o", obj + ".tmp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    os.replace(obj + ".tmp", obj)
    return obj


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    cpp, cu = sources()
    digest = _headers_digest()
    if force:
        for f in glob.glob(os.path.join(BUILD, "*.o")):
            os.remove(f)
    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(lambda s: _compile(s, digest), cpp + cu))
    # drop objects of older source versions (they would travel to the GPU box with the tree)
    keep = set(objs)
    for f in glob.glob(os.path.join(BUILD, "*.o")):
        if f not in keep:
            os.remove(f)
    stamp = hashlib.sha1("".join(objs).encode()).hexdigest()
    stamp_file = LIB + ".stamp"
    if os.path.exists(LIB) and os.path.exists(stamp_file) and open(stamp_file).read() == stamp:
        return LIB
    cmd = [NVCC] + ARCH + ["-shared", "-o", LIB + ".tmp"] + objs + ["-Xcompiler", "-fPIC", "-ldl", "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    os.replace(LIB + ".tmp", LIB)
    open(stamp_file, "w").write(stamp)
    if verbose:
        print("built", LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
