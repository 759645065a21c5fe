"""GPU tests of the shard layer (S9) on one B200: G logical shards (one tm_db
per shard on the same GPU) run the library's own split (tm_shard_counts) and
owner merge (tm_shard_merge) with device-to-device copies in place of NCCL
(loopback); the NCCL path itself runs with nranks = 1."""
import numpy as np
import pytest

import tmgen
from oracle import o2

pytestmark = pytest.mark.gpu
tmb = pytest.importorskip("paper_conf_eurosys_rogorapkmcc17_b200")
from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tm  # noqa: E402


class _CAI:
    def __init__(self, ptr, n, typestr="<u4"):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}


def _dev(torch, ptr, n, typestr="<u4"):
    if n == 0:
        return torch.zeros(0, dtype=torch.int32 if typestr == "<u4" else torch.int64, device="cuda")
    return torch.as_tensor(_CAI(ptr, n, typestr), device="cuda")


def _device_queries(torch, ts):
    t = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in
         (ts.vocab_bytes, ts.vocab_off.view(np.int64), ts.tag_idx.view(np.int32), ts.set_off.view(np.int64))]
    dq = tmb.device_tagsets(t[0].data_ptr(), t[1].data_ptr(), t[2].data_ptr(), t[3].data_ptr(),
                            ts.vocab_bytes.size, ts.vocab_off.size - 1, ts.tag_idx.size, ts.n_sets)
    return dq, t


@pytest.fixture(scope="module")
def wl():
    return tmgen.generate(20000, 2000, seed=31, max_partition=400)


@pytest.mark.parametrize("G", [2, 3, 5])
@pytest.mark.parametrize("unique", [False, True])
def test_loopback_sharded_equals_single(wl, G, unique):
    torch = pytest.importorskip("torch")
    dq, keep = _device_queries(torch, wl.queries)
    Q = wl.queries.n_sets
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition) as full:
        fq, fk = full.match_batch(wl.queries, unique)
        P_total = full.stats()["n_partitions"]
    shards = [tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, n_shards=G, shard=g)
              for g in range(G)]
    try:
        assert sum(s.stats()["n_partitions"] for s in shards) == P_total
        assert all(s.stats()["n_partitions_total"] == P_total for s in shards)
        # local match on every shard, cut at owner boundaries by the library
        segs = []
        for s in shards:
            s.match_batch_device(dq, unique)
            ptr, n = s.last_result()
            cnt = s.shard_counts(G)
            assert int(cnt.sum()) == n
            local = _dev(torch, ptr, n, "<u8").clone()
            off = np.concatenate([[0], np.cumsum(cnt)]).astype(np.int64)
            segs.append([local[off[g]:off[g + 1]] for g in range(G)])
        # loopback exchange + owner merge
        outq, outk = [], []
        for g, s in enumerate(shards):
            recv = torch.cat([segs[src][g] for src in range(G)]).contiguous()
            out = s.shard_merge(recv.data_ptr() if recv.numel() else 0, recv.numel(), Q, unique)
            q = _dev(torch, out.query, out.n).cpu().numpy().view(np.uint32)
            k = _dev(torch, out.key, out.n).cpu().numpy().view(np.uint32)
            lo, hi = tm.owner_range(Q, G, g)
            assert q.size == 0 or (q.min() >= lo and q.max() < hi)
            outq.append(q)
            outk.append(k)
        gq, gk = np.concatenate(outq), np.concatenate(outk)
        assert np.array_equal(gq, fq) and np.array_equal(gk, fk)
    finally:
        for s in shards:
            s.close()
    # and the single-handle result is the oracle's
    wq, wk = o2.match_brute(o2.encode(wl.db), wl.key_off, wl.keys, o2.encode(wl.queries), unique)
    assert np.array_equal(fq, wq) and np.array_equal(fk, wk)


@pytest.mark.parametrize("unique", [False, True])
def test_nccl_path_single_rank(wl, unique):
    """tm_comm_init + tm_match_batch_sharded_device (NCCL all-gather and
    grouped send/recv to self) == the unsharded device result."""
    torch = pytest.importorskip("torch")
    dq, keep = _device_queries(torch, wl.queries)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, n_shards=1, shard=0) as db:
        hq, hk = db.match_batch(wl.queries, unique)
        db.comm_init(tm.nccl_unique_id(), 1, 0)
        out = db.match_batch_sharded_device(dq, unique)
        q = _dev(torch, out.query, out.n).cpu().numpy().view(np.uint32)
        k = _dev(torch, out.key, out.n).cpu().numpy().view(np.uint32)
    assert np.array_equal(q, hq) and np.array_equal(k, hk)
