"""GPU tests of the multi-GPU modes that need no launcher on one B200:

* in-process multi-GPU databases (tm_config.n_gpus, device_ids; include/tagmatch.h): G
  sub-databases on device_ids = [0] * G (the same GPU: the peer copies of the exchange become
  device-to-device copies), partitioned and replicated, through
  tm_match_batch and tm_match_batch_csr, bit-exact against the oracle's brute force;
* the partition -> shard plan weighted by a routed query sample (tm_config.plan_sample);
* one-process-per-GPU replicated mode (n_shards > 1, shard_mode = replicated): each rank
  matches its owner range with no exchange; the slices concatenate to the global result.
"""
import numpy as np
import pytest

import tmgen
from oracle import o2

pytestmark = pytest.mark.gpu
tmb = pytest.importorskip("paper_conf_eurosys_rogorapkmcc17_b200")
from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tm  # noqa: E402


@pytest.fixture(scope="module")
def wl():
    return tmgen.generate(30000, 3000, seed=41, max_partition=600)


@pytest.fixture(scope="module")
def want(wl):
    db = o2.encode(wl.db)
    qs = o2.encode(wl.queries)
    return {u: o2.match_brute(db, wl.key_off, wl.keys, qs, u) for u in (False, True)}


def _eq(got, want, what):
    assert got[0].size == want[0].size, f"{what}: {got[0].size} pairs vs oracle {want[0].size}"
    assert np.array_equal(got[0], want[0]) and np.array_equal(got[1], want[1]), what


def _csr_to_pairs(off, key):
    q = np.repeat(np.arange(off.size - 1, dtype=np.uint32), np.diff(off).astype(np.int64))
    return q, key


@pytest.mark.parametrize("G", [2, 3])
@pytest.mark.parametrize("mode", [tm.TM_SHARD_PARTITIONED, tm.TM_SHARD_REPLICATED])
@pytest.mark.parametrize("tile_filter,row_order", [(1, 1), (0, 0)])
@pytest.mark.parametrize("fused", [True, False])
def test_in_process_group_equals_oracle(wl, want, G, mode, tile_filter, row_order, fused, monkeypatch):
    """Partitioned groups exchange through the fused scan emission (pairs stored into the owners'
    receive regions) or, with TM_NO_FUSED_EXCHANGE, through local merges + peer pulls."""
    if fused:
        monkeypatch.delenv("TM_NO_FUSED_EXCHANGE", raising=False)
    else:
        monkeypatch.setenv("TM_NO_FUSED_EXCHANGE", "1")
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=tile_filter,
                      row_order=row_order, n_gpus=G, shard_mode=mode, device_ids=[0] * G) as db:
        assert db.group_size() == G
        st = db.stats()
        assert st["n_gpus"] == G
        parts = [db.member_stats(g)["n_partitions"] for g in range(G)]
        total = db.member_stats(0)["n_partitions_total"]
        if mode == tm.TM_SHARD_PARTITIONED:
            assert sum(parts) == total and st["n_partitions"] == total
        else:
            assert all(p == total for p in parts)
        for unique in (False, True):
            for _ in range(2):   # second call: reused buffers
                _eq(db.match_batch(wl.queries, unique), want[unique], f"G={G} mode={mode} u={unique}")
            _eq(_csr_to_pairs(*db.match_batch_csr(wl.queries, unique)), want[unique], f"csr G={G} mode={mode}")
            st = db.stats()
            assert st["result_pairs"] == want[unique][0].size and st["n_queries"] == wl.queries.n_sets
            if mode == tm.TM_SHARD_REPLICATED:
                assert st["xchg_send_bytes"] == 0


@pytest.mark.parametrize("variant", ["", "13", "0", "6"])
def test_group_edge_batches(wl, want, variant, monkeypatch):
    """Empty batch, one query, fewer queries than GPUs (empty owner ranges), through the fused
    exchange of every emission path (filtered default, dense, no pre-check, streaming)."""
    if variant:
        monkeypatch.setenv("TM_SCAN_VARIANT", variant)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1, row_order=1,
                      n_gpus=3, device_ids=[0, 0, 0]) as db:
        for n in (0, 1, 2, 5):
            q = wl.queries.subset(np.arange(n))
            wq, wk = o2.match_brute(o2.encode(wl.db), wl.key_off, wl.keys, o2.encode(q), False) if n else \
                (np.zeros(0, np.uint32), np.zeros(0, np.uint32))
            _eq(db.match_batch(q, False), (wq, wk), f"n={n}")
            off, key = db.match_batch_csr(q, False)
            assert off.size == n + 1 and off[-1] == wq.size


def test_fused_exchange_region_overflow_retry(wl, want, monkeypatch):
    """Receive regions far too small for the first call: the scan's stores past the capacity are
    dropped, the counters report the overflow, the call re-runs with regions that fit."""
    monkeypatch.setenv("TM_FUSED_XCAP", "16")
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1, row_order=1,
                      n_gpus=3, device_ids=[0, 0, 0]) as db:
        for unique in (False, True):
            _eq(db.match_batch(wl.queries, unique), want[unique], f"overflow retry u={unique}")


def test_group_rejects_device_pointer_calls(wl):
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, n_gpus=2,
                      device_ids=[0, 0]) as db:
        with pytest.raises(tm.TagMatchError) as e:
            db.match_batch_device(tmb.device_tagsets(0, 0, 0, 0, 0, 0, 0, 0), False)
        assert e.value.status == -6   # TM_ESTATE
        with pytest.raises(tm.TagMatchError):
            db.partitions()


def test_plan_sample_balances_routed_work(wl, want):
    """with a routed query sample the plan weighs partitions by |P| x routed; the
    shards' candidate pairs (sum of |P| over routed (q, p)) on the full batch are then close to
    equal (the sample is the batch's first 1000 queries), and the result stays exact."""
    G = 3
    sample = wl.queries.subset(np.arange(1000))
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1, row_order=1,
                      n_gpus=G, device_ids=[0] * G, plan_sample=sample) as db:
        _eq(db.match_batch(wl.queries, False), want[False], "plan_sample")
        cand = np.array([db.member_stats(g)["candidate_pairs"] for g in range(G)], float)
        assert cand.max() / cand.mean() < 1.5, cand


@pytest.mark.parametrize("G", [2, 3])
def test_multiprocess_replicated_mode_slices(wl, want, G):
    """n_shards = G, shard_mode = replicated: rank g holds the whole table, matches owner range g
    of the (device-resident) batch with no exchange and no communicator."""
    torch = pytest.importorskip("torch")
    q = wl.queries
    t = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in
         (q.vocab_bytes, q.vocab_off.view(np.int64), q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
    dq = tmb.device_tagsets(t[0].data_ptr(), t[1].data_ptr(), t[2].data_ptr(), t[3].data_ptr(),
                            q.vocab_bytes.size, q.vocab_off.size - 1, q.tag_idx.size, q.n_sets)
    got_q, got_k = [], []
    for g in range(G):
        with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, n_shards=G, shard=g,
                          shard_mode=tm.TM_SHARD_REPLICATED) as db:
            out = db.match_batch_sharded_device(dq, False)
            lo, hi = tm.owner_range(q.n_sets, G, g)
            if out.n:
                qq = torch.as_tensor(_CAI(out.query, out.n), device="cuda").cpu().numpy().view(np.uint32)
                kk = torch.as_tensor(_CAI(out.key, out.n), device="cuda").cpu().numpy().view(np.uint32)
                assert qq.min() >= lo and qq.max() < hi
                got_q.append(qq.copy())
                got_k.append(kk.copy())
            assert db.stats()["xchg_send_bytes"] == 0
    _eq((np.concatenate(got_q), np.concatenate(got_k)), want[False], f"replicated G={G}")


class _CAI:
    def __init__(self, ptr, n, typestr="<u4"):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}
