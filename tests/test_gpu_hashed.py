"""Pre-hashed query input (tm_tagsets.vocab_hash: the throughput protocol
times pre-hashed query tags): the caller hashes each vocabulary string with FNV-1a-64 (reading
R1) and passes the hashes instead of the strings.  Matching must then be bit-exact with the
string input and with the oracle; the calls that keep strings reject it.

The test computes the hashes with the oracle's FNV-1a (o1.fnv1a64, pinned to the published
vectors in tests/golden/), so nothing on the expected side comes from the CUDA path.
"""
import numpy as np
import pytest

import tmgen
from oracle import o1, o2

pytestmark = pytest.mark.gpu

tmb = pytest.importorskip("paper_conf_eurosys_rogorapkmcc17_b200")


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_eurosys_rogorapkmcc17_b200 import _build
    _build.build()
    tmb.load()


def vocab_hashes(ts):
    vb, vo = ts.vocab_bytes, ts.vocab_off
    return np.array([o1.fnv1a64(bytes(vb[vo[v]:vo[v + 1]])) for v in range(vo.size - 1)], dtype=np.uint64)


@pytest.fixture(scope="module")
def wl():
    return tmgen.generate(20_000, 2_000, seed=41, max_partition=3_000)


def test_hashed_queries_match_strings_and_oracle(wl):
    q = wl.queries
    hq = tmb.HostTagSets.hashed(vocab_hashes(q), q.tag_idx, q.set_off)
    db_sig, q_sig = o2.encode(wl.db), o2.encode(q)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1,
                      row_order=1) as db:
        for unique in (False, True):
            gs = db.match_batch(q, unique)
            gh = db.match_batch(hq, unique)
            wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, q_sig, unique)
            assert np.array_equal(gh[0], wq) and np.array_equal(gh[1], wk), f"hashed vs oracle, unique={unique}"
            assert np.array_equal(gs[0], gh[0]) and np.array_equal(gs[1], gh[1])
        # the CSR host call and the device-pointer call take the hashes too
        off, keys = db.match_batch_csr(hq, False)
        wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, q_sig, False)
        assert np.array_equal(keys, wk) and np.array_equal(np.repeat(np.arange(q.n_sets), np.diff(off).astype(np.int64)), wq)
        torch = pytest.importorskip("torch")
        th = torch.from_numpy(vocab_hashes(q).view(np.int64)).cuda()
        tt = torch.from_numpy(np.ascontiguousarray(q.tag_idx).view(np.int32)).cuda()
        ts = torch.from_numpy(np.ascontiguousarray(q.set_off).view(np.int64)).cuda()
        dq = tmb.device_tagsets(0, 0, tt.data_ptr(), ts.data_ptr(), 0, th.numel(), tt.numel(), q.n_sets,
                                vocab_hash_ptr=th.data_ptr())
        out = db.match_batch_device(dq, False)
        assert out.n == wq.size


def test_hashed_identity_tags_and_encode(wl):
    """tag_idx NULL: the hashes are the tags themselves; tm_encode of hashes == the oracle encoder."""
    q = wl.queries.subset(np.arange(300))
    tags = [[bytes(q.vocab_bytes[q.vocab_off[v]:q.vocab_off[v + 1]]) for v in q.tag_idx[q.set_off[i]:q.set_off[i + 1]]]
            for i in range(q.n_sets)]
    flat = np.array([o1.fnv1a64(t) for ts in tags for t in ts], dtype=np.uint64)
    hq = tmb.HostTagSets.hashed(flat, None, q.set_off)
    got = tmb.encode(hq)
    want = np.array([o1.words(o1.encode(ts)) for ts in tags], dtype=np.uint64).reshape(-1, 3)
    assert np.array_equal(got, want)
    assert np.array_equal(tmb.encode(q), want)


def test_hashed_rejected_where_strings_are_needed(wl):
    q = wl.queries.subset(np.arange(50))
    hq = tmb.HostTagSets.hashed(vocab_hashes(q), q.tag_idx, q.set_off)
    with pytest.raises(tmb.TagMatchError):           # tm_build keeps the strings (exact mode, store)
        tmb.Database(hq, np.arange(q.n_sets + 1, dtype=np.uint64), np.arange(q.n_sets, dtype=np.uint32))
    both = tmb.HostTagSets.hashed(vocab_hashes(q), q.tag_idx, q.set_off)
    both.vb = np.ascontiguousarray(q.vocab_bytes, dtype=np.uint8)   # hashes AND strings: ambiguous
    both.c.vocab_bytes = both.vb.ctypes.data
    both.c.n_bytes = both.vb.size
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition) as db:
        with pytest.raises(tmb.TagMatchError):
            db.match_batch(both, False)
        db.match_batch(hq, False)                      # the handle stays usable
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, exact=1) as db:
        with pytest.raises(tmb.TagMatchError):           # the exact check compares strings
            db.match_batch(hq, False)
    # the mutable store interns tag strings (tm_add_sets), the stream replays strings
    mdb = tmb.Database.create(max_partition=1000)
    try:
        with pytest.raises(tmb.TagMatchError):
            mdb.add_sets(hq, np.arange(q.n_sets + 1, dtype=np.uint64), np.arange(q.n_sets, dtype=np.uint32))
    finally:
        mdb.close()
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition) as db:
        st = tmb.tagmatch.Stream(db, 64, 1000, False)
        try:
            with pytest.raises(tmb.TagMatchError):
                st.replay(hq, np.zeros(q.n_sets, np.uint64))
        finally:
            st.close()


@pytest.mark.parametrize("mode", [0, 1])   # TM_SHARD_PARTITIONED, TM_SHARD_REPLICATED
def test_hashed_queries_in_process_group(wl, mode):
    """An in-process multi-GPU database (2 sub-databases on device 0) takes the hashed batch and
    a hashed plan sample (partition -> GPU plan by routed counts) and returns the oracle's pairs."""
    q = wl.queries
    hq = tmb.HostTagSets.hashed(vocab_hashes(q), q.tag_idx, q.set_off)
    smp = q.subset(np.arange(500))
    hs = tmb.HostTagSets.hashed(vocab_hashes(smp), smp.tag_idx, smp.set_off)
    db_sig, q_sig = o2.encode(wl.db), o2.encode(q)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1, row_order=1,
                      n_gpus=2, shard_mode=mode, device_ids=[0, 0], plan_sample=hs) as db:
        for unique in (False, True):
            gq, gk = db.match_batch(hq, unique)
            wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, q_sig, unique)
            assert np.array_equal(gq, wq) and np.array_equal(gk, wk), f"mode={mode} unique={unique}"
