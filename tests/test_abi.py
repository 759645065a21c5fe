"""C-ABI library: builds, loads, exports every declared symbol, fails loudly
without a GPU (no CPU fallback), and never touches the oracle.  CPU only."""
import ctypes
import glob
import os
import re

import numpy as np
import pytest

import paper_conf_eurosys_rogorapkmcc17_b200 as tmb
from paper_conf_eurosys_rogorapkmcc17_b200 import _build, tagmatch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "tagmatch.h")


@pytest.fixture(scope="module")
def lib():
    _build.build()
    return tagmatch.load()


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(tm_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for n in ["tm_build", "tm_match_batch", "tm_free", "tm_pairs_free", "tm_match_batch_device", "tm_encode",
              "tm_stats"]:
        assert n in names
    assert sorted(tagmatch.EXPORTS) == names


def test_library_exports_every_declared_symbol(lib):
    for n in declared_functions():
        assert hasattr(lib, n), n
    assert lib.tm_abi_version() == 5
    # the symbols are real exports of the in-tree .so (nm -D)
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", tagmatch.LIB_PATH], capture_output=True, text=True).stdout
    for n in declared_functions():
        assert re.search(rf"\bT {n}$", out, re.M), n


def test_built_for_sm100a(lib):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", tagmatch.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_strerror(lib):
    assert lib.tm_strerror(0) == b"ok"
    assert lib.tm_strerror(-1) == b"invalid argument"
    assert lib.tm_strerror(-3) == b"CUDA error"


def test_invalid_arguments_rejected_before_device_use(lib):
    ts = tagmatch.HostTagSets(np.frombuffer(b"ab", np.uint8), np.array([0, 1, 2], np.uint64),
                              np.array([0, 5], np.uint32), np.array([0, 2], np.uint64))
    h = ctypes.c_void_p()
    st = lib.tm_build(ctypes.byref(ts.c), None, None, None, ctypes.byref(h))
    assert st == -1 and b"tag_idx out of range" in lib.tm_last_error()
    bad = tagmatch.HostTagSets(np.frombuffer(b"ab", np.uint8), np.array([0, 1, 2], np.uint64),
                               np.array([0, 1], np.uint32), np.array([0, 2, 1], np.uint64))
    bad.c.n_tags = 1
    st = lib.tm_build(ctypes.byref(bad.c), None, None, None, ctypes.byref(h))
    assert st == -1
    assert lib.tm_build(None, None, None, None, ctypes.byref(h)) == -1


@pytest.mark.skipif(os.path.exists("/dev/nvidia0"), reason="checks the no-GPU behaviour")
def test_no_gpu_fails_loudly(lib):
    """Without a CUDA device the library returns TM_ECUDA: there is no CPU fallback."""
    ts = tagmatch.HostTagSets(np.frombuffer(b"ab", np.uint8), np.array([0, 1, 2], np.uint64),
                              np.array([0, 1], np.uint32), np.array([0, 2], np.uint64))
    with pytest.raises(tmb.TagMatchError) as e:
        tmb.Database(ts, keys=np.array([7], np.uint32))
    assert e.value.status == -3
    with pytest.raises(tmb.TagMatchError):
        tmb.encode(ts)


def test_product_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_eurosys_rogorapkmcc17_b200")
    for f in glob.glob(os.path.join(pkg, "**", "*.*"), recursive=True):
        if f.endswith((".py", ".cu", ".cpp", ".h")):
            src = open(f).read()
            assert not re.search(r"\boracle\b|o2\.c|liboracle|\bo1\b", src), f
