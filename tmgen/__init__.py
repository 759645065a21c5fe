"""Seeded synthetic workload generator (shared by oracle and library tests/bench).

Holds none of TagMatch's arithmetic (no hashing, encoding or matching): it only
draws tag ids / keys / queries shaped like the paper's Twitter workload
(sec. 4.2) and marshals them into the C-ABI's interned
CSR form (vocabulary strings + per-set tag indices).  See tmgen/gen.c and the
"Input recipe" section of DESIGN.md.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_SO = os.path.join(_HERE, "libtmgen.so")
_lib = None

UINT32_MAX = 0xFFFFFFFF

# BASELINE.json configs.  max_partition: UINT32_MAX = a
# single mask-empty partition (C1 "single partition set"), else MAX_P = 200K
# (PAPER.md:371).
CONFIGS = {
    "C1": dict(n_sets=10_000, n_queries=1_000, seed=1, max_partition=UINT32_MAX, total_tags=0),
    "C2": dict(n_sets=1_000_000, n_queries=100_000, seed=2, max_partition=200_000, total_tags=0),
    "C3": dict(n_sets=100_000_000, n_queries=1_000_000, seed=3, max_partition=200_000, total_tags=0),
    "C4": dict(n_sets=300_000_000, n_queries=1_000_000, seed=4, max_partition=200_000, total_tags=0),
}
# C5: one 100M-set database (seed 500), query batches of exactly t tags (query seed 500 + t)
for _t in range(2, 21, 2):
    CONFIGS[f"C5t{_t}"] = dict(n_sets=100_000_000, n_queries=100_000, seed=500, query_seed=500 + _t,
                               max_partition=200_000, total_tags=_t)


def build_lib(force: bool = False) -> str:
    """Compile gen.c into libtmgen.so (plain -O2, no -march: the .so travels to the GPU box)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread",
                               "-D_GNU_SOURCE", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build_lib())
        vp, u64, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int
        L.tg_db_generate.restype = vp
        L.tg_db_generate.argtypes = [u64, u64, i32]
        L.tg_db_free.argtypes = [vp]
        for f in ("tg_db_n_sets", "tg_db_n_tags", "tg_db_n_keys", "tg_db_n_users"):
            getattr(L, f).restype = u64
            getattr(L, f).argtypes = [vp]
        L.tg_db_copy.argtypes = [vp, vp, vp, vp, vp, vp]
        L.tg_queries_generate.restype = vp
        L.tg_queries_generate.argtypes = [vp, u64, u64, i32, i32, i32, i32]
        L.tg_q_free.argtypes = [vp]
        L.tg_q_n.restype = u64
        L.tg_q_n.argtypes = [vp]
        L.tg_q_n_tags.restype = u64
        L.tg_q_n_tags.argtypes = [vp]
        L.tg_q_copy.argtypes = [vp, vp, vp, vp]
        L.tg_strings_size.restype = u64
        L.tg_strings_size.argtypes = [vp, u64]
        L.tg_strings.argtypes = [vp, u64, vp, vp]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data) if a.size else None


@dataclass
class TagSets:
    """A batch of tag sets in the ABI's interned CSR form (see include/tagmatch.h).

    set i = strings vocab[tag_idx[set_off[i]:set_off[i+1]]], where string v is
    vocab_bytes[vocab_off[v]:vocab_off[v+1]].
    """
    vocab_bytes: np.ndarray  # uint8
    vocab_off: np.ndarray    # uint64 [n_vocab+1]
    tag_idx: np.ndarray      # uint32 [n_tags]
    set_off: np.ndarray      # uint64 [n_sets+1]

    @property
    def n_sets(self) -> int:
        return int(self.set_off.size - 1)

    def strings(self, i: int) -> list[bytes]:
        """The tag strings of set i (small-case helper for the Python oracle)."""
        vb = self.vocab_bytes.tobytes() if not hasattr(self, "_vb") else self._vb
        self._vb = vb
        out = []
        for t in self.tag_idx[self.set_off[i]:self.set_off[i + 1]]:
            out.append(vb[self.vocab_off[t]:self.vocab_off[t + 1]])
        return out

    def subset(self, idx: np.ndarray) -> "TagSets":
        """Sets idx (in that order), same vocabulary."""
        idx = np.asarray(idx, dtype=np.int64)
        lens = (self.set_off[idx + 1] - self.set_off[idx]).astype(np.uint64)
        off = np.zeros(idx.size + 1, dtype=np.uint64)
        np.cumsum(lens, out=off[1:])
        parts = [self.tag_idx[self.set_off[i]:self.set_off[i + 1]] for i in idx]
        tags = np.concatenate(parts).astype(np.uint32) if parts else np.zeros(0, np.uint32)
        return TagSets(self.vocab_bytes, self.vocab_off, tags, off)


def tag_strings(ids: np.ndarray) -> tuple[np.ndarray, np.ndarray]:
    """Strings of global tag ids: '<lang>_t<rank>' or 'u<publisher>'."""
    L = lib()
    ids = np.ascontiguousarray(ids, dtype=np.uint32)
    nbytes = L.tg_strings_size(_p(ids), ids.size)
    b = np.zeros(max(int(nbytes), 1), dtype=np.uint8)
    off = np.zeros(ids.size + 1, dtype=np.uint64)
    L.tg_strings(_p(ids), ids.size, ctypes.c_void_p(b.ctypes.data), ctypes.c_void_p(off.ctypes.data))
    return b[:int(nbytes)], off


def intern(set_off: np.ndarray, tags: np.ndarray) -> TagSets:
    """CSR of global tag ids -> interned form with a compact vocabulary."""
    tags = np.ascontiguousarray(tags, dtype=np.uint32)
    if tags.size == 0:
        uniq, inv = np.zeros(0, np.uint32), np.zeros(0, np.uint32)
    else:
        # dense remap (ids are < 8*2^20 + publishers): O(n), no sort
        present = np.zeros(int(tags.max()) + 1, dtype=bool)
        present[tags] = True
        uniq = np.flatnonzero(present).astype(np.uint32)
        remap = np.cumsum(present, dtype=np.int64) - 1
        inv = remap[tags].astype(np.uint32)
    vb, vo = tag_strings(uniq)
    return TagSets(vb, vo, inv, np.ascontiguousarray(set_off, dtype=np.uint64))


@dataclass
class Workload:
    name: str
    db: TagSets              # N unique tag sets
    key_off: np.ndarray      # uint64 [N+1]: set i's keys = keys[key_off[i]:key_off[i+1]]
    keys: np.ndarray         # uint32 [K]
    queries: TagSets         # Q queries
    query_base: np.ndarray   # uint64 [Q]: the DB set each query was built from
    max_partition: int
    db_ids: np.ndarray | None = None   # global tag ids (generator-internal)
    q_ids: np.ndarray | None = None


def generate(n_sets: int, n_queries: int, seed: int, extra: tuple[int, int] = (2, 4),
             total_tags: int = 0, max_partition: int = 200_000, nthreads: int = 0,
             name: str = "custom", keep_ids: bool = False, query_seed: int | None = None) -> Workload:
    L = lib()
    h = L.tg_db_generate(seed, n_sets, nthreads)
    try:
        n = L.tg_db_n_sets(h)
        nt = L.tg_db_n_tags(h)
        nk = L.tg_db_n_keys(h)
        set_off = np.zeros(n + 1, np.uint64)
        tags = np.zeros(nt, np.uint32)
        key_off = np.zeros(n + 1, np.uint64)
        keys = np.zeros(nk, np.uint32)
        L.tg_db_copy(h, _p(set_off), _p(tags), _p(key_off), _p(keys), None)
        qs = seed + (1 << 32) if query_seed is None else query_seed
        qh = L.tg_queries_generate(h, qs, n_queries, extra[0], extra[1], total_tags, nthreads)
        try:
            nq = L.tg_q_n(qh)
            nqt = L.tg_q_n_tags(qh)
            q_off = np.zeros(nq + 1, np.uint64)
            q_tags = np.zeros(nqt, np.uint32)
            base = np.zeros(nq, np.uint64)
            L.tg_q_copy(qh, _p(q_off), _p(q_tags), _p(base))
        finally:
            L.tg_q_free(qh)
    finally:
        L.tg_db_free(h)
    wl = Workload(name, intern(set_off, tags), key_off, keys, intern(q_off, q_tags), base, max_partition)
    if keep_ids:
        wl.db_ids, wl.q_ids = tags, q_tags
    return wl


def _zipf_draw(rng: np.random.Generator, cdf: np.ndarray, shape) -> np.ndarray:
    return np.searchsorted(cdf, rng.random(shape), side="right").astype(np.uint32)


def generate_crafted(n_sets: int, set_tags: int, query_tags: int, n_queries: int, seed: int,
                     vocab: int = 1 << 20, max_partition: int = 200_000, name: str = "crafted",
                     query_seed: int | None = None) -> Workload:
    """The scaled-down second workload of sec. 4.4: every DB set has exactly
    `set_tags` distinct tags (2 or 3), every query has exactly `query_tags` tags (6-10) = one DB
    set (its base) plus query_tags - set_tags extra tags.  Tags are drawn from
    a Zipf(1) vocabulary of `vocab` ids (the popularity law of the Twitter workload,
    PAPER.md:264); DB sets are distinct; one key per set (key = set index).  numpy PCG64, seeded."""
    assert 1 <= set_tags <= query_tags and vocab <= (1 << 20)
    rng = np.random.Generator(np.random.PCG64(seed))
    w = 1.0 / np.arange(1, vocab + 1, dtype=np.float64)
    cdf = np.cumsum(w) / w.sum()
    cdf[-1] = 1.0
    assert set_tags <= 3, "sets are deduplicated as one packed u64 (3 x 20-bit ids)"
    packed = np.zeros(0, np.uint64)
    while packed.size < n_sets:
        d = np.sort(_zipf_draw(rng, cdf, (int((n_sets - packed.size) * 1.3) + 64, set_tags)), axis=1)
        d = d[np.all(d[:, 1:] != d[:, :-1], axis=1)].astype(np.uint64)
        p = np.zeros(d.shape[0], np.uint64)
        for c in range(set_tags):
            p = (p << np.uint64(20)) | d[:, c]
        packed = np.sort(np.concatenate([packed, p]))
        packed = packed[np.concatenate(([True], packed[1:] != packed[:-1]))]
    packed = packed[rng.permutation(packed.size)[:n_sets]]
    rows = np.zeros((n_sets, set_tags), np.uint32)
    for c in range(set_tags - 1, -1, -1):
        rows[:, c] = (packed & np.uint64(0xFFFFF)).astype(np.uint32)
        packed = packed >> np.uint64(20)
    set_off = np.arange(n_sets + 1, dtype=np.uint64) * np.uint64(set_tags)
    key_off = np.arange(n_sets + 1, dtype=np.uint64)
    keys = np.arange(n_sets, dtype=np.uint32)
    rng = np.random.Generator(np.random.PCG64(seed + (1 << 32) if query_seed is None else query_seed))
    base = rng.integers(0, n_sets, n_queries).astype(np.uint64)
    e = query_tags - set_tags
    q = np.zeros((n_queries, query_tags), np.uint32)
    q[:, :set_tags] = rows[base]
    todo = np.arange(n_queries)
    while todo.size and e:
        q[todo, set_tags:] = _zipf_draw(rng, cdf, (todo.size, e))
        s = np.sort(q[todo], axis=1)
        todo = todo[np.any(s[:, 1:] == s[:, :-1], axis=1)]
    q_off = np.arange(n_queries + 1, dtype=np.uint64) * np.uint64(query_tags)
    return Workload(name, intern(set_off, rows.reshape(-1)), key_off, keys, intern(q_off, q.reshape(-1)),
                    base, max_partition)


# sec. 4.4 crafted workloads: C6 = the paper's hardest case, 2-tag sets and
# 10-tag queries over the largest DB of Fig. 10 (5M sets; "more than 32,000 queries per second",
# PAPER.md:395); C7 = the Fig. 11 workload, 3M sets of 3 tags, 6-tag queries.
CRAFTED = {
    "C6": dict(n_sets=5_000_000, set_tags=2, query_tags=10, n_queries=100_000, seed=6),
    "C7": dict(n_sets=3_000_000, set_tags=3, query_tags=6, n_queries=100_000, seed=7),
}


def config(name: str, **overrides) -> Workload:
    if name in CRAFTED:
        c = dict(CRAFTED[name])
        c.update(overrides)
        return generate_crafted(c["n_sets"], c["set_tags"], c["query_tags"], c["n_queries"], c["seed"],
                                max_partition=c.get("max_partition", 200_000), name=name,
                                query_seed=c.get("query_seed"))
    c = dict(CONFIGS[name])
    c.update(overrides)
    return generate(c["n_sets"], c["n_queries"], c["seed"], total_tags=c["total_tags"],
                    max_partition=c["max_partition"], name=name, query_seed=c.get("query_seed"))


def generate_sweep(n_sets: int, seed: int, n_queries: int, totals, query_seed_base: int,
                   max_partition: int = 200_000, nthreads: int = 0):
    """One database and one query batch per total tag count t (C5):
    returns (Workload with the t = totals[0] batch, {t: TagSets}, {t: base indices})."""
    L = lib()
    h = L.tg_db_generate(seed, n_sets, nthreads)
    try:
        n, nt, nk = L.tg_db_n_sets(h), L.tg_db_n_tags(h), L.tg_db_n_keys(h)
        set_off = np.zeros(n + 1, np.uint64)
        tags = np.zeros(nt, np.uint32)
        key_off = np.zeros(n + 1, np.uint64)
        keys = np.zeros(nk, np.uint32)
        L.tg_db_copy(h, _p(set_off), _p(tags), _p(key_off), _p(keys), None)
        batches, bases = {}, {}
        for t in totals:
            qh = L.tg_queries_generate(h, query_seed_base + t, n_queries, 0, 0, t, nthreads)
            try:
                nq, nqt = L.tg_q_n(qh), L.tg_q_n_tags(qh)
                q_off = np.zeros(nq + 1, np.uint64)
                q_tags = np.zeros(nqt, np.uint32)
                base = np.zeros(nq, np.uint64)
                L.tg_q_copy(qh, _p(q_off), _p(q_tags), _p(base))
            finally:
                L.tg_q_free(qh)
            batches[t], bases[t] = intern(q_off, q_tags), base
    finally:
        L.tg_db_free(h)
    t0 = list(totals)[0]
    wl = Workload(f"sweep{n_sets}", intern(set_off, tags), key_off, keys, batches[t0], bases[t0], max_partition)
    return wl, batches, bases
