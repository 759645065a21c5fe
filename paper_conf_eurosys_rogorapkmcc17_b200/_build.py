"""Build libtagmatch.so in-tree with nvcc for sm_100a (B200).

Usage: python -m paper_conf_eurosys_rogorapkmcc17_b200._build [--force] [--verbose-ptxas]
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
BUILD = os.path.join(ROOT, "build", "obj")
LIB = os.path.join(PKG, "libtagmatch.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> str:
    """nccl.h of the NCCL that torch uses (pip nvidia-nccl); the library dlopens libnccl at run time."""
    try:
        import nvidia.nccl
        for d in nvidia.nccl.__path__:
            inc = os.path.join(d, "include")
            if os.path.exists(os.path.join(inc, "nccl.h")):
                return inc
    except Exception:
        pass
    return "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/include"


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _deps():
    return _sources() + glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(INCLUDE, "tagmatch.h"),
                                                                os.path.abspath(__file__)]


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in _deps())


def build_id() -> str:
    """sha256 (16 hex) of every library source: identifies the kernels a profile was taken on."""
    import hashlib
    h = hashlib.sha256()
    for d in sorted(_deps()):
        if d.endswith("_build.py"):
            continue
        h.update(os.path.basename(d).encode())
        with open(d, "rb") as f:
            h.update(f.read())
    return h.hexdigest()[:16]


def _compile(src: str, verbose_ptxas: bool, bid: str) -> str:
    obj = os.path.join(BUILD, os.path.basename(src) + ".o")
    cmd = [NVCC, "-c", src, "-o", obj, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-I", INCLUDE, "-I", CSRC, "-I", _nccl_include(),
           "-Xcompiler", "-fPIC,-O3,-Wall", "--expt-relaxed-constexpr", "-DNDEBUG",
           f"-DTM_BUILD_ID=\"{bid}\""]
    cmd += os.environ.get("TM_NVCC_FLAGS", "").split()  # experiments only (e.g. -DTM_BLOCK_TILES=4)
    if verbose_ptxas and src.endswith(".cu"):
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    if verbose_ptxas:
        sys.stderr.write(r.stderr)
    return obj


def build(force: bool = False, verbose_ptxas: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    os.makedirs(BUILD, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=8) as ex:
        bid = build_id()
        objs = list(ex.map(lambda s: _compile(s, verbose_ptxas, bid), _sources()))
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC, "-shared", *ARCH, "-o", tmp, *objs, "-Xcompiler", "-fPIC", "-lpthread", "-ldl"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, LIB)
    return LIB


def build_tools() -> str:
    """Measurement tools (not the product): build/int_peak from scripts/int_peak.cu, the INT/logic
    pipe microbenchmark whose result is bench.py's roofline peak."""
    src = os.path.join(ROOT, "scripts", "int_peak.cu")
    exe = os.path.join(ROOT, "build", "int_peak")
    if os.path.exists(exe) and os.path.getmtime(exe) >= os.path.getmtime(src):
        return exe
    os.makedirs(os.path.dirname(exe), exist_ok=True)
    r = subprocess.run([NVCC, "-O3", *ARCH, "-lineinfo", "-o", exe + ".tmp", src], capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    os.replace(exe + ".tmp", exe)
    return exe


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose_ptxas="--verbose-ptxas" in sys.argv))
