"""ctypes binding of ORACLE O2 (oracle/o2.c).  TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
--impl reference) may import this module.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "o2.c")
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build_lib(force: bool = False) -> str:
    """gcc -O2 (no -march: the .so travels to the GPU box's host)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread",
                               "-D_GNU_SOURCE", _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build_lib())
        vp, u64, i32, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint32
        L.o2_fnv1a64.restype = u64
        L.o2_fnv1a64.argtypes = [vp, u64]
        L.o2_splitmix_mix.restype = u64
        L.o2_splitmix_mix.argtypes = [u64]
        L.o2_tag_positions.argtypes = [vp, u64, vp]
        L.o2_encode.argtypes = [vp, vp, vp, vp, u64, vp, i32]
        L.o2_match_brute.restype = vp
        L.o2_match_brute.argtypes = [vp, vp, vp, u64, vp, vp, u64, i32, i32]
        L.o2_result_n.restype = u64
        L.o2_result_n.argtypes = [vp]
        L.o2_result_copy.argtypes = [vp, vp, vp]
        L.o2_result_free.argtypes = [vp]
        L.o2_alg1.restype = vp
        L.o2_alg1.argtypes = [vp, u64, u32]
        L.o2_index_n_parts.restype = u64
        L.o2_index_n_parts.argtypes = [vp]
        L.o2_index_copy.argtypes = [vp, vp, vp, vp]
        L.o2_index_free.argtypes = [vp]
        L.o2_match_partitioned.restype = vp
        L.o2_match_partitioned.argtypes = [vp, vp, vp, vp, vp, vp, u64, i32, i32, vp]
        L.o2_fp_montecarlo.argtypes = [u64, i32, i32, u64, i32, vp]
        L.o2_threads.restype = i32
        L.o2_threads.argtypes = [i32]
        _lib = L
    return _lib


def _p(a):
    if a is None:
        return None
    return ctypes.c_void_p(a.ctypes.data) if a.size else ctypes.c_void_p(0)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def threads(n: int = 0) -> int:
    return lib().o2_threads(n)


def fnv1a64(b: bytes) -> int:
    buf = np.frombuffer(b, dtype=np.uint8) if b else np.zeros(1, np.uint8)
    return int(lib().o2_fnv1a64(_p(buf), len(b)))


def splitmix_mix(x: int) -> int:
    return int(lib().o2_splitmix_mix(x))


def tag_positions(b: bytes) -> list[int]:
    buf = np.frombuffer(b, dtype=np.uint8) if b else np.zeros(1, np.uint8)
    out = np.zeros(7, np.uint32)
    lib().o2_tag_positions(_p(buf), len(b), _p(out))
    return [int(x) for x in out]


def encode(ts, nthreads: int = 0) -> np.ndarray:
    """Signatures [n_sets, 3] uint64 of a TagSets-like object (vocab_bytes,
    vocab_off, tag_idx (or None), set_off)."""
    vb = _c(ts.vocab_bytes, np.uint8)
    if vb.size == 0:
        vb = np.zeros(1, np.uint8)
    vo = _c(ts.vocab_off, np.uint64)
    ti = None if ts.tag_idx is None else _c(ts.tag_idx, np.uint32)
    so = _c(ts.set_off, np.uint64)
    n = so.size - 1
    out = np.zeros((max(n, 0), 3), np.uint64)
    if n > 0:
        lib().o2_encode(_p(vb), _p(vo), _p(ti) if ti is not None and ti.size else None, _p(so), n, _p(out), nthreads)
    return out


def _result(h):
    L = lib()
    try:
        n = L.o2_result_n(h)
        q = np.zeros(n, np.uint32)
        k = np.zeros(n, np.uint32)
        if n:
            L.o2_result_copy(h, _p(q), _p(k))
    finally:
        L.o2_result_free(h)
    return q, k


def match_brute(db_sig, key_off, keys, q_sig, unique: bool, qid=None, nthreads: int = 0):
    """Brute force over every DB entry (the definition)."""
    db = _c(db_sig, np.uint64).reshape(-1, 3)
    ko = _c(key_off, np.uint64)
    ks = _c(keys, np.uint32)
    qs = _c(q_sig, np.uint64).reshape(-1, 3)
    qi = None if qid is None else _c(qid, np.uint32)
    h = lib().o2_match_brute(_p(db), _p(ko), _p(ks), db.shape[0], _p(qs), _p(qi) if qi is not None else None,
                             qs.shape[0], int(unique), nthreads)
    return _result(h)


class Index:
    """Algorithm 1 partition table computed by O2."""

    def __init__(self, db_sig, max_p: int):
        L = lib()
        self.db = _c(db_sig, np.uint64).reshape(-1, 3)
        self.h = L.o2_alg1(_p(self.db), self.db.shape[0], max_p)
        P = L.o2_index_n_parts(self.h)
        self.masks = np.zeros((P, 3), np.uint64)
        self.part_off = np.zeros(P + 1, np.uint64)
        self.members = np.zeros(self.db.shape[0], np.uint64)
        if P:
            L.o2_index_copy(self.h, _p(self.masks), _p(self.part_off), _p(self.members))

    @property
    def n_parts(self) -> int:
        return self.masks.shape[0]

    def match(self, key_off, keys, q_sig, unique: bool, qid=None, nthreads: int = 0):
        """Alg. 2 routing + linear scan of each routed partition; returns (q, k, stats)
        with stats = (routed (q, partition) pairs, pair checks)."""
        ko = _c(key_off, np.uint64)
        ks = _c(keys, np.uint32)
        qs = _c(q_sig, np.uint64).reshape(-1, 3)
        qi = None if qid is None else _c(qid, np.uint32)
        st = np.zeros(2, np.uint64)
        h = lib().o2_match_partitioned(self.h, _p(self.db), _p(ko), _p(ks), _p(qs),
                                       _p(qi) if qi is not None else None, qs.shape[0], int(unique),
                                       nthreads, _p(st))
        q, k = _result(h)
        return q, k, (int(st[0]), int(st[1]))

    def close(self):
        if self.h:
            lib().o2_index_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def fp_montecarlo(seed: int, s2: int, d: int, trials: int, nthreads: int = 0) -> tuple[int, int]:
    """(false positives, total popcount of sig(S2)) over `trials` (PAPER.md:132 fn.3)."""
    out = np.zeros(2, np.uint64)
    lib().o2_fp_montecarlo(seed, s2, d, trials, nthreads, _p(out))
    return int(out[0]), int(out[1])
