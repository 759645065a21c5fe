"""Thin ctypes binding of libtagmatch.so (include/tagmatch.h).

Argument marshalling only: every step of the matching path runs in the
library's CUDA kernels.  There is no CPU fallback -- if the extension is
missing or no B200 is visible, calls raise.

Names follow the ABI: tm_build / tm_match_batch / tm_match_batch_device /
tm_free / tm_encode / tm_stats / tm_partitions.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libtagmatch.so")

TM_DEFAULT_MAX_PARTITION = 200_000
TM_NO_PARTITIONING = 0xFFFFFFFF
TM_AUTO_MAX_PARTITION = 0xFFFFFFFE
STATUS = {0: "TM_OK", -1: "TM_EINVAL", -2: "TM_ENOMEM", -3: "TM_ECUDA", -4: "TM_ENCCL", -5: "TM_ERANGE",
          -6: "TM_ESTATE"}


class TagMatchError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS.get(status, status)}: {detail}")
        self.status = status


class tm_tagsets(ctypes.Structure):
    _fields_ = [("vocab_bytes", ctypes.c_void_p), ("vocab_off", ctypes.c_void_p), ("tag_idx", ctypes.c_void_p),
                ("set_off", ctypes.c_void_p), ("n_bytes", ctypes.c_uint64), ("n_vocab", ctypes.c_uint64),
                ("n_tags", ctypes.c_uint64), ("n_sets", ctypes.c_uint64), ("vocab_hash", ctypes.c_void_p)]


class tm_config(ctypes.Structure):
    _fields_ = [("max_partition", ctypes.c_uint32), ("device", ctypes.c_int32), ("n_shards", ctypes.c_uint32),
                ("shard", ctypes.c_uint32), ("tile_filter", ctypes.c_uint32), ("row_order", ctypes.c_uint32),
                ("exact", ctypes.c_uint32), ("n_gpus", ctypes.c_uint32), ("shard_mode", ctypes.c_uint32),
                ("reserved", ctypes.c_uint32), ("device_ids", ctypes.c_void_p),
                ("plan_sample", ctypes.POINTER(tm_tagsets))]


TM_SHARD_PARTITIONED = 0
TM_SHARD_REPLICATED = 1


class tm_pairs(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint64), ("query", ctypes.POINTER(ctypes.c_uint32)),
                ("key", ctypes.POINTER(ctypes.c_uint32)), ("priv_", ctypes.c_void_p)]


class tm_csr(ctypes.Structure):
    _fields_ = [("n_queries", ctypes.c_uint64), ("n", ctypes.c_uint64), ("q_off", ctypes.POINTER(ctypes.c_uint64)),
                ("key", ctypes.POINTER(ctypes.c_uint32)), ("priv_", ctypes.c_void_p)]


class tm_dev_pairs(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint64), ("query", ctypes.c_void_p), ("key", ctypes.c_void_p)]


class tm_stream_config(ctypes.Structure):
    _fields_ = [("max_batch", ctypes.c_uint32), ("timeout_us", ctypes.c_uint32), ("unique", ctypes.c_int32),
                ("reserved", ctypes.c_uint32)]


class tm_stream_result(ctypes.Structure):
    _fields_ = [("n_queries", ctypes.c_uint64), ("tickets", ctypes.POINTER(ctypes.c_uint64)),
                ("submit_ns", ctypes.POINTER(ctypes.c_uint64)), ("key_off", ctypes.POINTER(ctypes.c_uint64)),
                ("keys", ctypes.POINTER(ctypes.c_uint32)), ("dispatch_ns", ctypes.c_uint64),
                ("done_ns", ctypes.c_uint64), ("priv_", ctypes.c_void_p)]


class tm_stats_t(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in
                ("n_sets", "n_entries", "n_unique", "n_rows", "n_partitions", "n_partitions_total")] + \
               [("build_ms", ctypes.c_double)] + \
               [(n, ctypes.c_uint64) for n in
                ("n_queries", "routed", "candidate_pairs", "tile_tests", "pair_checks", "matched_sets",
                 "emitted_pairs", "result_pairs", "work_items", "retries")] + \
               [(n, ctypes.c_double) for n in ("encode_ms", "route_ms", "scan_ms", "merge_ms", "total_ms")] + \
               [("scan_launches", ctypes.c_uint32), ("kernel_launches", ctypes.c_uint32),
                ("exact_checked", ctypes.c_uint64), ("exact_kept", ctypes.c_uint64),
                ("scan_variant", ctypes.c_uint32), ("tuning", ctypes.c_uint32),
                ("xchg_send_bytes", ctypes.c_uint64), ("xchg_recv_bytes", ctypes.c_uint64),
                ("xchg_ms", ctypes.c_double), ("local_ms", ctypes.c_double),
                ("max_partition", ctypes.c_uint32), ("n_gpus", ctypes.c_uint32)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


EXPORTS = ["tm_build", "tm_match_batch", "tm_match_batch_csr", "tm_match_batch_device", "tm_pairs_free",
           "tm_csr_free", "tm_free", "tm_strerror",
           "tm_last_error", "tm_abi_version", "tm_build_id", "tm_encode", "tm_stats", "tm_partitions", "tm_partition_sigs",
           "tm_owner_range", "tm_shard_plan", "tm_exchange_plan", "tm_group_size", "tm_group_member", "tm_partition_host", "tm_last_result", "tm_shard_counts",
           "tm_shard_merge", "tm_nccl_unique_id", "tm_comm_init", "tm_match_batch_sharded_device",
           "tm_stream_open", "tm_stream_submit", "tm_stream_poll", "tm_stream_result_free", "tm_stream_flush",
           "tm_stream_replay", "tm_stream_close", "tm_create", "tm_add_set", "tm_remove_set", "tm_add_sets",
           "tm_consolidate", "tm_pending"]

_lib = None


def load(path: str = LIB_PATH):
    """Load the in-tree library.  Raises if it is missing: there is no fallback."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not built: run __graft_entry__.build() "
                          "(python -m paper_conf_eurosys_rogorapkmcc17_b200._build)")
    L = ctypes.CDLL(path)
    vp, P = ctypes.c_void_p, ctypes.POINTER
    L.tm_build.restype = ctypes.c_int
    L.tm_build.argtypes = [P(tm_tagsets), vp, vp, P(tm_config), P(vp)]
    L.tm_match_batch.restype = ctypes.c_int
    L.tm_match_batch.argtypes = [vp, P(tm_tagsets), ctypes.c_int, P(tm_pairs)]
    L.tm_match_batch_device.restype = ctypes.c_int
    L.tm_match_batch_device.argtypes = [vp, P(tm_tagsets), ctypes.c_int, P(tm_dev_pairs), vp]
    L.tm_pairs_free.argtypes = [P(tm_pairs)]
    L.tm_match_batch_csr.restype = ctypes.c_int
    L.tm_match_batch_csr.argtypes = [vp, P(tm_tagsets), ctypes.c_int, P(tm_csr)]
    L.tm_csr_free.argtypes = [P(tm_csr)]
    L.tm_free.argtypes = [vp]
    L.tm_strerror.restype = ctypes.c_char_p
    L.tm_strerror.argtypes = [ctypes.c_int]
    L.tm_last_error.restype = ctypes.c_char_p
    L.tm_abi_version.restype = ctypes.c_uint32
    L.tm_build_id.restype = ctypes.c_char_p
    L.tm_encode.restype = ctypes.c_int
    L.tm_encode.argtypes = [P(tm_tagsets), vp, ctypes.c_int]
    L.tm_stats.restype = ctypes.c_int
    L.tm_stats.argtypes = [vp, P(tm_stats_t)]
    L.tm_partitions.restype = ctypes.c_int
    L.tm_partitions.argtypes = [vp, vp, vp]
    L.tm_partition_sigs.restype = ctypes.c_int
    L.tm_partition_sigs.argtypes = [vp, ctypes.c_uint64, vp]
    u64, u32, i32 = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
    for name, args in [("tm_owner_range", [u64, u32, u32, vp, vp]),
                       ("tm_shard_plan", [vp, vp, vp, u64, u32, vp]),
                       ("tm_exchange_plan", [vp, u32, u32, vp, vp]),
                       ("tm_group_size", [vp, vp]),
                       ("tm_group_member", [vp, u32, vp]),
                       ("tm_partition_host", [vp, u64, u32, vp, vp, vp, vp, vp]),
                       ("tm_last_result", [vp, vp, vp]),
                       ("tm_shard_counts", [vp, u32, vp]),
                       ("tm_shard_merge", [vp, vp, u64, u64, i32, P(tm_dev_pairs), vp]),
                       ("tm_nccl_unique_id", [vp, u64]),
                       ("tm_comm_init", [vp, vp, u64, i32, i32]),
                       ("tm_match_batch_sharded_device", [vp, P(tm_tagsets), i32, P(tm_dev_pairs), vp])]:
        getattr(L, name).restype = ctypes.c_int
        getattr(L, name).argtypes = args
    for name, args in [("tm_stream_open", [vp, P(tm_stream_config), P(vp)]),
                       ("tm_stream_submit", [vp, vp, vp, u64, P(ctypes.c_uint64)]),
                       ("tm_stream_poll", [vp, i32, P(tm_stream_result)]),
                       ("tm_stream_flush", [vp]),
                       ("tm_stream_replay", [vp, P(tm_tagsets), vp])]:
        getattr(L, name).restype = ctypes.c_int
        getattr(L, name).argtypes = args
    for name, args in [("tm_create", [P(tm_config), P(vp)]),
                       ("tm_add_set", [vp, vp, vp, u64, u32]),
                       ("tm_remove_set", [vp, vp, vp, u64, u32]),
                       ("tm_add_sets", [vp, P(tm_tagsets), vp, vp]),
                       ("tm_consolidate", [vp]),
                       ("tm_pending", [vp, vp, vp])]:
        getattr(L, name).restype = ctypes.c_int
        getattr(L, name).argtypes = args
    L.tm_stream_result_free.argtypes = [P(tm_stream_result)]
    L.tm_stream_close.argtypes = [vp]
    _lib = L
    return L


def _check(st: int):
    if st != 0:
        raise TagMatchError(st, load().tm_last_error().decode(errors="replace"))


def _ptr(a):
    if a is None:
        return None
    return ctypes.c_void_p(a.ctypes.data) if a.size else None


class HostTagSets:
    """Host-side tm_tagsets; keeps the numpy arrays alive while referenced."""

    def __init__(self, vocab_bytes, vocab_off, tag_idx, set_off):
        self.vb = np.ascontiguousarray(vocab_bytes, dtype=np.uint8)
        self.vo = np.ascontiguousarray(vocab_off, dtype=np.uint64)
        self.ti = None if tag_idx is None else np.ascontiguousarray(tag_idx, dtype=np.uint32)
        self.so = np.ascontiguousarray(set_off, dtype=np.uint64)
        n_tags = int(self.so[-1]) if self.so.size else 0
        self.c = tm_tagsets(_ptr(self.vb), _ptr(self.vo), _ptr(self.ti) if self.ti is not None else None,
                            _ptr(self.so), self.vb.size, max(self.vo.size - 1, 0), n_tags, max(self.so.size - 1, 0))

    @classmethod
    def of(cls, ts):
        """From any object with vocab_bytes / vocab_off / tag_idx / set_off (e.g. tmgen.TagSets)."""
        return cls(ts.vocab_bytes, ts.vocab_off, ts.tag_idx, ts.set_off)

    @classmethod
    def hashed(cls, vocab_hash, tag_idx, set_off):
        """A pre-hashed vocabulary (tm_tagsets.vocab_hash: FNV-1a-64 of each vocabulary string, the
        caller's own hashing; no strings are passed)."""
        self = cls.__new__(cls)
        self.vh = np.ascontiguousarray(vocab_hash, dtype=np.uint64)
        self.vb = self.vo = None
        self.ti = None if tag_idx is None else np.ascontiguousarray(tag_idx, dtype=np.uint32)
        self.so = np.ascontiguousarray(set_off, dtype=np.uint64)
        n_tags = int(self.so[-1]) if self.so.size else 0
        self.c = tm_tagsets(None, None, _ptr(self.ti) if self.ti is not None else None, _ptr(self.so), 0,
                            self.vh.size, n_tags, max(self.so.size - 1, 0), _ptr(self.vh))
        return self


def device_tagsets(vocab_bytes_ptr, vocab_off_ptr, tag_idx_ptr, set_off_ptr, n_bytes, n_vocab, n_tags, n_sets,
                   vocab_hash_ptr=0):
    """tm_tagsets of device pointers (ints, e.g. torch tensor data_ptr()); vocab_hash_ptr: a
    pre-hashed vocabulary instead of vocab_bytes / vocab_off."""
    return tm_tagsets(vocab_bytes_ptr or None, vocab_off_ptr or None, tag_idx_ptr or None, set_off_ptr or None,
                      n_bytes, n_vocab, n_tags, n_sets, vocab_hash_ptr or None)


def make_config(max_partition=0, device=-1, n_shards=1, shard=0, tile_filter=0, row_order=0,
                exact=0, n_gpus=0, shard_mode=0) -> tm_config:
    c = tm_config()
    c.max_partition = max_partition
    c.device = device
    c.n_shards = n_shards
    c.shard = shard
    c.tile_filter = tile_filter
    c.row_order = row_order
    c.exact = exact
    c.n_gpus = n_gpus
    c.shard_mode = shard_mode
    return c


class Database:
    """A tm_db handle: tm_build on construction, tm_free on close()."""

    def __init__(self, sets, key_off=None, keys=None, max_partition=0, device=-1, n_shards=1, shard=0,
                 tile_filter=0, row_order=0, exact=0, n_gpus=0, shard_mode=0, device_ids=None, plan_sample=None):
        """n_gpus > 1: an in-process multi-GPU database on device_ids (default 0..n_gpus-1; repeats
        allowed); shard_mode TM_SHARD_PARTITIONED / TM_SHARD_REPLICATED; plan_sample: host query
        batch whose routing weighs the partition -> shard plan."""
        L = load()
        self._sets = sets if isinstance(sets, HostTagSets) else HostTagSets.of(sets)
        self._ko = None if key_off is None else np.ascontiguousarray(key_off, dtype=np.uint64)
        self._ks = np.ascontiguousarray(keys if keys is not None else np.zeros(0), dtype=np.uint32)
        cfg = make_config(max_partition, device, n_shards, shard, tile_filter, row_order, exact, n_gpus, shard_mode)
        ids = None
        if device_ids is not None:
            ids = np.ascontiguousarray(device_ids, dtype=np.int32)
            cfg.device_ids = ctypes.c_void_p(ids.ctypes.data)
        smp = None
        if plan_sample is not None:
            smp = plan_sample if isinstance(plan_sample, HostTagSets) else HostTagSets.of(plan_sample)
            cfg.plan_sample = ctypes.pointer(smp.c)
        h = ctypes.c_void_p()
        _check(L.tm_build(ctypes.byref(self._sets.c), _ptr(self._ko), _ptr(self._ks) if self._ks.size else None,
                          ctypes.byref(cfg), ctypes.byref(h)))
        self.h = h
        del self._sets, ids, smp  # inputs are not retained by the library

    @classmethod
    def create(cls, max_partition=0, device=-1, tile_filter=0, row_order=0, exact=0, n_gpus=0, shard_mode=0,
               device_ids=None):
        """tm_create: an empty mutable database (add_set / remove_set, then consolidate; Table 2)."""
        self = cls.__new__(cls)
        cfg = make_config(max_partition, device, 1, 0, tile_filter, row_order, exact, n_gpus, shard_mode)
        ids = None
        if device_ids is not None:
            ids = np.ascontiguousarray(device_ids, dtype=np.int32)
            cfg.device_ids = ctypes.c_void_p(ids.ctypes.data)
        h = ctypes.c_void_p()
        _check(load().tm_create(ctypes.byref(cfg), ctypes.byref(h)))
        self.h = h
        return self

    @staticmethod
    def _tags(tags):
        b = b"".join(tags)
        off = np.zeros(len(tags) + 1, np.uint64)
        if tags:
            off[1:] = np.cumsum([len(t) for t in tags])
        buf = np.frombuffer(b, np.uint8) if b else np.zeros(1, np.uint8)
        return buf, off

    def add_set(self, tags: list[bytes], key: int):
        buf, off = self._tags(tags)
        _check(load().tm_add_set(self.h, _ptr(buf), _ptr(off), len(tags), key))

    def remove_set(self, tags: list[bytes], key: int):
        buf, off = self._tags(tags)
        _check(load().tm_remove_set(self.h, _ptr(buf), _ptr(off), len(tags), key))

    def add_sets(self, sets, key_off=None, keys=None):
        s = sets if isinstance(sets, HostTagSets) else HostTagSets.of(sets)
        ko = None if key_off is None else np.ascontiguousarray(key_off, dtype=np.uint64)
        ks = np.ascontiguousarray(keys if keys is not None else np.zeros(0), dtype=np.uint32)
        _check(load().tm_add_sets(self.h, ctypes.byref(s.c), _ptr(ko) if ko is not None else None,
                                  _ptr(ks) if ks.size else None))

    def consolidate(self):
        _check(load().tm_consolidate(self.h))

    def pending(self) -> tuple[int, int]:
        """(staged operations, live entry instances) of a mutable handle."""
        a, b = ctypes.c_uint64(), ctypes.c_uint64()
        _check(load().tm_pending(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def match_batch(self, queries, unique: bool) -> tuple[np.ndarray, np.ndarray]:
        """tm_match_batch: host queries -> sorted (query, key) arrays (copies out of pinned memory)."""
        L = load()
        q = queries if isinstance(queries, HostTagSets) else HostTagSets.of(queries)
        out = tm_pairs()
        _check(L.tm_match_batch(self.h, ctypes.byref(q.c), int(bool(unique)), ctypes.byref(out)))
        try:
            n = out.n
            if n:
                qa = np.ctypeslib.as_array(out.query, shape=(n,)).copy()
                ka = np.ctypeslib.as_array(out.key, shape=(n,)).copy()
            else:
                qa = np.zeros(0, np.uint32)
                ka = np.zeros(0, np.uint32)
        finally:
            L.tm_pairs_free(ctypes.byref(out))
        return qa, ka

    def match_batch_csr(self, queries, unique: bool) -> tuple[np.ndarray, np.ndarray]:
        """tm_match_batch_csr: host queries -> (q_off [Q+1] uint64, key [n] uint32) per-query key lists."""
        L = load()
        q = queries if isinstance(queries, HostTagSets) else HostTagSets.of(queries)
        out = tm_csr()
        _check(L.tm_match_batch_csr(self.h, ctypes.byref(q.c), int(bool(unique)), ctypes.byref(out)))
        try:
            off = np.ctypeslib.as_array(out.q_off, shape=(out.n_queries + 1,)).copy()
            key = np.ctypeslib.as_array(out.key, shape=(out.n,)).copy() if out.n else np.zeros(0, np.uint32)
        finally:
            L.tm_csr_free(ctypes.byref(out))
        return off, key

    def match_batch_csr_raw(self, queries: HostTagSets, unique: bool) -> tm_csr:
        """tm_match_batch_csr returning the library-owned pinned tm_csr (caller must free_csr)."""
        out = tm_csr()
        _check(load().tm_match_batch_csr(self.h, ctypes.byref(queries.c), int(bool(unique)), ctypes.byref(out)))
        return out

    @staticmethod
    def free_csr(c: tm_csr):
        load().tm_csr_free(ctypes.byref(c))

    def match_batch_raw(self, queries: HostTagSets, unique: bool) -> tm_pairs:
        """tm_match_batch returning the library-owned pinned tm_pairs (caller must free_pairs)."""
        out = tm_pairs()
        _check(load().tm_match_batch(self.h, ctypes.byref(queries.c), int(bool(unique)), ctypes.byref(out)))
        return out

    @staticmethod
    def free_pairs(p: tm_pairs):
        load().tm_pairs_free(ctypes.byref(p))

    def match_batch_device(self, dq: tm_tagsets, unique: bool, stream: int = 0) -> tm_dev_pairs:
        """tm_match_batch_device: device-resident queries; result stays in device memory."""
        out = tm_dev_pairs()
        _check(load().tm_match_batch_device(self.h, ctypes.byref(dq), int(bool(unique)), ctypes.byref(out),
                                            ctypes.c_void_p(stream) if stream else None))
        return out

    def group_size(self) -> int:
        n = ctypes.c_uint32()
        _check(load().tm_group_size(self.h, ctypes.byref(n)))
        return n.value

    def member_stats(self, g: int) -> dict:
        """tm_stats of sub-database g of an in-process multi-GPU handle (tm_group_member)."""
        sub = ctypes.c_void_p()
        _check(load().tm_group_member(self.h, g, ctypes.byref(sub)))
        s = tm_stats_t()
        _check(load().tm_stats(sub, ctypes.byref(s)))
        return s.as_dict()

    def stats(self) -> dict:
        s = tm_stats_t()
        _check(load().tm_stats(self.h, ctypes.byref(s)))
        return s.as_dict()

    def partitions(self) -> tuple[np.ndarray, np.ndarray]:
        n = self.stats()["n_partitions"]
        masks = np.zeros((n, 3), np.uint64)
        sizes = np.zeros(n, np.uint64)
        if n:
            _check(load().tm_partitions(self.h, _ptr(masks), _ptr(sizes)))
        return masks, sizes

    def partition_sigs(self, p: int, size: int) -> np.ndarray:
        out = np.zeros((size, 3), np.uint64)
        if size:
            _check(load().tm_partition_sigs(self.h, p, _ptr(out)))
        return out

    # ---- shard layer (include/tagmatch.h "shards")
    def last_result(self) -> tuple[int, int]:
        """(device pointer, n) of the last call's sorted (q<<32|key) pairs."""
        ptr, n = ctypes.c_void_p(), ctypes.c_uint64()
        _check(load().tm_last_result(self.h, ctypes.byref(ptr), ctypes.byref(n)))
        return ptr.value or 0, n.value

    def shard_counts(self, n_owners: int) -> np.ndarray:
        out = np.zeros(n_owners, np.uint64)
        _check(load().tm_shard_counts(self.h, n_owners, _ptr(out)))
        return out

    def shard_merge(self, pairs_ptr: int, n: int, n_queries: int, unique: bool, stream: int = 0) -> tm_dev_pairs:
        out = tm_dev_pairs()
        _check(load().tm_shard_merge(self.h, ctypes.c_void_p(pairs_ptr) if pairs_ptr else None, n, n_queries,
                                     int(bool(unique)), ctypes.byref(out),
                                     ctypes.c_void_p(stream) if stream else None))
        return out

    def comm_init(self, uid: bytes, nranks: int, rank: int):
        buf = ctypes.create_string_buffer(uid, len(uid))
        _check(load().tm_comm_init(self.h, buf, len(uid), nranks, rank))

    def match_batch_sharded_device(self, dq: tm_tagsets, unique: bool, stream: int = 0) -> tm_dev_pairs:
        out = tm_dev_pairs()
        _check(load().tm_match_batch_sharded_device(self.h, ctypes.byref(dq), int(bool(unique)), ctypes.byref(out),
                                                    ctypes.c_void_p(stream) if stream else None))
        return out

    def close(self):
        if getattr(self, "h", None):
            load().tm_free(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def encode(sets, device: int = -1) -> np.ndarray:
    """tm_encode: Bloom signatures [n_sets, 3] uint64 computed on the GPU."""
    L = load()
    s = sets if isinstance(sets, HostTagSets) else HostTagSets.of(sets)
    n = s.c.n_sets
    out = np.zeros((n, 3), np.uint64)
    _check(L.tm_encode(ctypes.byref(s.c), _ptr(out), device))
    return out


def abi_version() -> int:
    return int(load().tm_abi_version())


def build_id() -> str:
    """tm_build_id: hash of the sources the loaded library was compiled from."""
    return load().tm_build_id().decode()


# ------------------------------------------------------------ shard layer --
def owner_range(n_queries: int, n_owners: int, owner: int) -> tuple[int, int]:
    lo, hi = ctypes.c_uint64(), ctypes.c_uint64()
    _check(load().tm_owner_range(n_queries, n_owners, owner, ctypes.byref(lo), ctypes.byref(hi)))
    return lo.value, hi.value


def shard_plan(masks: np.ndarray, sizes: np.ndarray, n_shards: int, routed: np.ndarray | None = None) -> np.ndarray:
    """tm_shard_plan: contiguous partition ranges of ~equal work |P| x routed (or |P| x 4^-|mask|)."""
    masks = np.ascontiguousarray(masks, dtype=np.uint64).reshape(-1, 3)
    sizes = np.ascontiguousarray(sizes, dtype=np.uint64)
    r = None if routed is None else np.ascontiguousarray(routed, dtype=np.uint64)
    out = np.zeros(masks.shape[0], np.uint32)
    _check(load().tm_shard_plan(_ptr(masks), _ptr(sizes), _ptr(r) if r is not None else None, masks.shape[0],
                                n_shards, _ptr(out)))
    return out


def exchange_plan(counts: np.ndarray, rank: int) -> tuple[np.ndarray, np.ndarray]:
    """tm_exchange_plan: (send_off [G+1], recv_off [G+1]) of `rank` from the G x G count matrix
    counts[s, d] = pairs rank s holds for owner d."""
    c = np.ascontiguousarray(counts, dtype=np.uint64)
    G = c.shape[0]
    so = np.zeros(G + 1, np.uint64)
    ro = np.zeros(G + 1, np.uint64)
    _check(load().tm_exchange_plan(_ptr(c), G, rank, _ptr(so), _ptr(ro)))
    return so, ro


def partition_host(sigs: np.ndarray, max_partition: int = 0):
    """Algorithm 1 on the host (no GPU): (masks [P,3], sizes [P], distinct sigs [U,3] partition by partition)."""
    sigs = np.ascontiguousarray(sigs, dtype=np.uint64).reshape(-1, 3)
    n = max(sigs.shape[0], 1)
    masks = np.zeros((n, 3), np.uint64)
    sizes = np.zeros(n, np.uint64)
    out = np.zeros((n, 3), np.uint64)
    P, U = ctypes.c_uint64(), ctypes.c_uint64()
    _check(load().tm_partition_host(_ptr(sigs), sigs.shape[0], max_partition, _ptr(masks), _ptr(sizes), _ptr(out),
                                    ctypes.byref(P), ctypes.byref(U)))
    return masks[:P.value], sizes[:P.value], out[:U.value]


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(load().tm_nccl_unique_id(buf, 128))
    return buf.raw


# -------------------------------------------------------------- streaming --
class Stream:
    """tm_stream: one-query submissions batched by size or timeout."""

    def __init__(self, db: Database, max_batch: int, timeout_us: int, unique: bool):
        cfg = tm_stream_config(max_batch, timeout_us, int(bool(unique)), 0)
        h = ctypes.c_void_p()
        _check(load().tm_stream_open(db.h, ctypes.byref(cfg), ctypes.byref(h)))
        self.h = h
        self._db = db

    def submit(self, tags: list[bytes]) -> int:
        b = b"".join(tags)
        off = np.zeros(len(tags) + 1, np.uint64)
        off[1:] = np.cumsum([len(t) for t in tags]) if tags else []
        buf = np.frombuffer(b, np.uint8) if b else np.zeros(1, np.uint8)
        t = ctypes.c_uint64()
        _check(load().tm_stream_submit(self.h, _ptr(buf), _ptr(off), len(tags), ctypes.byref(t)))
        return t.value

    def replay(self, queries, arrival_ns: np.ndarray):
        q = queries if isinstance(queries, HostTagSets) else HostTagSets.of(queries)
        arr = np.ascontiguousarray(arrival_ns, dtype=np.uint64)
        _check(load().tm_stream_replay(self.h, ctypes.byref(q.c), _ptr(arr)))

    def flush(self):
        _check(load().tm_stream_flush(self.h))

    def poll(self, wait: bool = True):
        """Next completed batch as a dict of numpy arrays, or None."""
        r = tm_stream_result()
        _check(load().tm_stream_poll(self.h, int(bool(wait)), ctypes.byref(r)))
        if r.n_queries == 0:
            return None
        n = r.n_queries
        try:
            ko = np.ctypeslib.as_array(r.key_off, shape=(n + 1,)).copy()
            out = {"tickets": np.ctypeslib.as_array(r.tickets, shape=(n,)).copy(),
                   "submit_ns": np.ctypeslib.as_array(r.submit_ns, shape=(n,)).copy(),
                   "key_off": ko,
                   "keys": np.ctypeslib.as_array(r.keys, shape=(int(ko[-1]),)).copy() if ko[-1] else
                   np.zeros(0, np.uint32),
                   "dispatch_ns": r.dispatch_ns, "done_ns": r.done_ns}
        finally:
            load().tm_stream_result_free(ctypes.byref(r))
        return out

    def close(self):
        if getattr(self, "h", None):
            load().tm_stream_close(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
