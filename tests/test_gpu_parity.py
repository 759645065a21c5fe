"""GPU parity: the CUDA path (through the C ABI) vs the oracle, element by
element, on seeded inputs.  Bit-exact: this is integer / bitwise work, and the
output is the canonically sorted (query, key) pair list.

Run with `pytest -m gpu` on a B200.
"""
import random

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


def assert_pairs_equal(got, want, what=""):
    gq, gk = got
    wq, wk = want
    assert gq.size == wq.size, f"{what}: {gq.size} pairs vs oracle {wq.size}"
    bad = np.nonzero((gq != wq) | (gk != wk))[0]
    assert bad.size == 0, f"{what}: first mismatch at {bad[:5]}: got {gq[bad[0]], gk[bad[0]]} want {wq[bad[0]], wk[bad[0]]}"


def oracle_pairs(wl, unique, qsel=None, brute=True, max_p=50_000):
    db = o2.encode(wl.db)
    qs = o2.encode(wl.queries)
    qid = None
    if qsel is not None:
        qs = qs[qsel]
        qid = np.asarray(qsel, np.uint32)
    if brute:
        return o2.match_brute(db, wl.key_off, wl.keys, qs, unique, qid=qid)
    q, k, _ = o2.Index(db, max_p).match(wl.key_off, wl.keys, qs, unique, qid=qid)
    return q, k


def tagsets(strings_per_set, vocab=None):
    """Build a tmgen.TagSets from python lists of byte strings (direct form)."""
    flat = [t for s in strings_per_set for t in s]
    vb = np.frombuffer(b"".join(flat), np.uint8) if flat and any(flat) else np.zeros(0, np.uint8)
    vo = np.zeros(len(flat) + 1, np.uint64)
    vo[1:] = np.cumsum([len(t) for t in flat]) if flat else []
    so = np.zeros(len(strings_per_set) + 1, np.uint64)
    so[1:] = np.cumsum([len(s) for s in strings_per_set]) if strings_per_set else []
    return tmgen.TagSets(vb, vo, np.arange(len(flat), dtype=np.uint32), so)


# ------------------------------------------------------------------ encoder --
def test_encode_bit_exact_c1(c1):
    got = tmb.encode(c1.db)
    want = o2.encode(c1.db)
    assert np.array_equal(got, want)
    gq = tmb.encode(c1.queries)
    assert np.array_equal(gq, o2.encode(c1.queries))


def test_encode_special_strings():
    rnd = random.Random(5)
    sets = [[b""], [b"cat"], [b"fr_cat", b"cat"], [b"u123", b"u123"], [bytes(range(256))],
            [bytes(rnd.getrandbits(8) for _ in range(rnd.randrange(0, 70))) for _ in range(rnd.randrange(0, 9))]]
    sets += [[bytes(rnd.getrandbits(8) for _ in range(rnd.randrange(0, 30))) for _ in range(rnd.randrange(0, 6))]
             for _ in range(300)]
    ts = tagsets(sets)
    got = tmb.encode(ts)
    for i, s in enumerate(sets):
        assert tuple(int(x) for x in got[i]) == o1.words(o1.encode(s)), i


# ----------------------------------------------------------------- matching --
@pytest.mark.parametrize("unique", [False, True])
@pytest.mark.parametrize("tile_filter", [0, 1, 2])
def test_c1_single_partition(c1, unique, tile_filter):
    """BASELINE config 0: 10k sets, 1k queries, one mask-empty partition."""
    want = oracle_pairs(c1, unique)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=c1.max_partition, tile_filter=tile_filter) as db:
        got = db.match_batch(c1.queries, unique)
        st = db.stats()
    assert_pairs_equal(got, want, "C1")
    assert st["n_partitions"] == 1 and st["routed"] == c1.queries.n_sets
    assert st["candidate_pairs"] == c1.queries.n_sets * c1.db.n_sets
    if tile_filter == 2:
        assert st["pair_checks"] == st["candidate_pairs"]


@pytest.mark.parametrize("unique", [False, True])
@pytest.mark.parametrize("tile_filter", [1, 2])
def test_c1_balanced_row_order(c1, unique, tile_filter):
    """Row order 1 (reading R18: balanced splits inside partitions) with AND
    masks: same result (the order inside a partition is lossless)."""
    want = oracle_pairs(c1, unique)
    for max_p in (0xFFFFFFFF, 2000):
        with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=max_p, tile_filter=tile_filter,
                          row_order=1) as db:
            got = db.match_batch(c1.queries, unique)
        assert_pairs_equal(got, want, f"C1 row_order=1 MAX_P={max_p}")


def test_row_order_needs_and_masks(c1):
    with pytest.raises(tmb.TagMatchError):
        tmb.Database(c1.db, c1.key_off, c1.keys, tile_filter=0, row_order=1)


@pytest.mark.parametrize("nq", [1, 2, 3, 4, 5, 8, 9, 40])
@pytest.mark.parametrize("max_p", [0xFFFFFFFF, 500])
@pytest.mark.parametrize("layout", [(0, 0), (1, 1)])
def test_small_batches(c1, nq, max_p, layout):
    """Batches of <= 8 routed queries take the unfiltered streaming path (<= 4: direct check
    over 128-row units, 5-8: the two-word pre-check), in the streaming-only kernels when the
    whole call has <= 8 queries; 9 and 40 straddle it (per partition).  MAX_P 500 makes
    partitions whose padded row counts are not multiples of the unit."""
    qsel = np.arange(0, c1.queries.n_sets, c1.queries.n_sets // nq)[:nq]
    q = c1.queries.subset(qsel)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=max_p, tile_filter=layout[0],
                      row_order=layout[1]) as db:
        for unique in (False, True):
            got = db.match_batch(q, unique)
            want = o2.match_brute(o2.encode(c1.db), c1.key_off, c1.keys, o2.encode(q), unique)
            assert_pairs_equal(got, want, f"nq={nq}")
            if nq <= 8:
                assert db.stats()["scan_variant"] == (6 if nq <= 4 else 7)


@pytest.mark.parametrize("max_p", [200_000, 1000, 64, 1])
def test_c1_metamorphic_max_partition(c1, max_p):
    """The result is invariant under MAX_P (partitioning is lossless)."""
    want = oracle_pairs(c1, False)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=max_p) as db:
        got = db.match_batch(c1.queries, False)
    assert_pairs_equal(got, want, f"C1 MAX_P={max_p}")


@pytest.mark.parametrize("max_p", [500, 2000])
def test_partition_table_matches_oracle_alg1(c1, max_p):
    """Library Alg. 1 == O2 Alg. 1 (same FIFO acceptance order, masks, members)."""
    db_sig = o2.encode(c1.db)
    ix = o2.Index(db_sig, max_p)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=max_p) as db:
        st = db.stats()
        assert st["n_unique"] == c1.db.n_sets  # no signature collisions in C1
        masks, sizes = db.partitions()
        assert masks.shape[0] == ix.n_parts
        assert np.array_equal(masks, ix.masks)
        for p in range(ix.n_parts):
            mem = ix.members[ix.part_off[p]:ix.part_off[p + 1]].astype(np.int64)
            want = db_sig[mem]
            want = want[np.lexsort((want[:, 2], want[:, 1], want[:, 0]))]
            got = db.partition_sigs(p, int(sizes[p]))
            assert np.array_equal(got, want), p  # members, lexicographically sorted


@pytest.fixture(scope="module")
def c2():
    return tmgen.config("C2")


@pytest.fixture(scope="module")
def c2_oracle(c2):
    return {u: oracle_pairs(c2, u, brute=False, max_p=50_000) for u in (False, True)}


@pytest.mark.parametrize("max_p,row_order", [(500, 0), (2000, 1), (1, 0), (0xFFFFFFFF, 1), (64, 1)])
def test_gpu_build_equals_host_build(c1, max_p, row_order, monkeypatch):
    """consolidate() on the GPU (tm_build.cu, depth-synchronous Alg. 1) builds the
    same table as the host implementation (FIFO queue): partitions in the same
    order, same masks, same rows in the same order."""
    def table(host):
        if host:
            monkeypatch.setenv("TM_BUILD_HOST", "1")
        else:
            monkeypatch.delenv("TM_BUILD_HOST", raising=False)
        with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=max_p, tile_filter=1,
                          row_order=row_order) as db:
            masks, sizes = db.partitions()
            sigs = [db.partition_sigs(p, int(sizes[p])) for p in range(sizes.size)]
            st = db.stats()
            q, k = db.match_batch(c1.queries, False)
        return masks, sizes, sigs, st, q, k
    gm, gs, gsig, gst, gq, gk = table(False)
    hm, hs, hsig, hst, hq, hk = table(True)
    assert np.array_equal(gm, hm) and np.array_equal(gs, hs)
    assert all(np.array_equal(a, b) for a, b in zip(gsig, hsig))
    for k_ in ("n_unique", "n_rows", "n_entries", "n_partitions"):
        assert gst[k_] == hst[k_], k_
    assert np.array_equal(gq, hq) and np.array_equal(gk, hk)


@pytest.mark.parametrize("layout", [(0, 0), (1, 1)], ids=["paper", "balanced"])
def test_c2_full_parity(c2, c2_oracle, layout):
    """BASELINE config 1: 1M sets, 100k queries, MAX_P = 200K; the oracle
    uses MAX_P = 50K so no partitioning misreading can hide.  Both layouts:
    lexicographic + Alg. 4 prefix, and balanced splits + AND masks."""
    wl = c2
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=layout[0],
                      row_order=layout[1]) as db:
        for unique in (False, True):
            got = db.match_batch(wl.queries, unique)
            assert_pairs_equal(got, c2_oracle[unique], f"C2 unique={unique}")
    # every query matches at least its base set
    assert np.unique(got[0]).size == wl.queries.n_sets


@pytest.mark.parametrize("variant", ["0", "5", "6", "7", "8", "9", "10", "11", "12", "13",
                                     "14", "15", "16", "17", "18"])
def test_c2_every_scan_variant(c2, c2_oracle, variant, monkeypatch):
    """Every scan-kernel variant (TM_SCAN_VARIANT) gives the oracle's
    pairs at C2, in the layout bench.py times (balanced splits + AND masks)."""
    monkeypatch.setenv("TM_SCAN_VARIANT", variant)
    wl = c2
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1,
                      row_order=1) as db:
        for unique in (False, True):
            got = db.match_batch(wl.queries, unique)
            assert_pairs_equal(got, c2_oracle[unique], f"C2 variant={variant} unique={unique}")
            # the streaming-only kernels (6, 7) cannot take a filtered call: they map to 0 / 5
            assert db.stats()["scan_variant"] == {"6": 0, "7": 5}.get(variant, int(variant))


def test_c2_sampled_against_brute_force(c2):
    """The partitioned oracle is itself pinned to brute force on a query sample."""
    wl = c2
    rnd = np.random.default_rng(12)
    qsel = np.sort(rnd.choice(wl.queries.n_sets, 512, replace=False))
    want = oracle_pairs(wl, False, qsel=qsel, brute=True)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition) as db:
        gq, gk = db.match_batch(wl.queries, False)
    keep = np.isin(gq, qsel)
    assert_pairs_equal((gq[keep], gk[keep]), want, "C2 sample")


# ------------------------------------------------------------- edge cases --
def _edge_db():
    """Empty sets, duplicates with different keys, repeated tags, ragged sizes."""
    rnd = random.Random(17)
    vocab = [f"t{i}".encode() for i in range(60)] + [b"", b"\xff\x00z"]
    sets, keys = [], []
    for i in range(1000):
        s = [rnd.choice(vocab) for _ in range(rnd.randint(0, 6))]
        sets.append(s)
        keys.append([rnd.randrange(50) for _ in range(rnd.randint(0, 3))])
    sets += [[], [], [b"t1", b"t1", b"t2"], [b"t2", b"t1"]]   # duplicates -> merged signatures
    keys += [[7, 7], [8], [9], [9]]
    queries = [[rnd.choice(vocab) for _ in range(rnd.randint(0, 14))] for _ in range(333)]
    queries += [[], vocab, [b"zzz"]]
    return sets, keys, queries


@pytest.mark.parametrize("max_p", [0xFFFFFFFF, 50, 1])
@pytest.mark.parametrize("unique", [False, True])
def test_edge_cases(max_p, unique):
    sets, keys, queries = _edge_db()
    db_ts, q_ts = tagsets(sets), tagsets(queries)
    key_off = np.zeros(len(keys) + 1, np.uint64)
    key_off[1:] = np.cumsum([len(k) for k in keys])
    flat = np.array([k for kl in keys for k in kl], np.uint32)
    want = o1.match([o1.encode(s) for s in sets], keys, [o1.encode(q) for q in queries], unique)
    with tmb.Database(db_ts, key_off, flat, max_partition=max_p) as db:
        gq, gk = db.match_batch(q_ts, unique)
        st = db.stats()
    assert list(zip(gq.tolist(), gk.tolist())) == want
    assert st["n_unique"] < len(sets)   # identical signatures merged (reading R10)


def test_empty_inputs():
    one = tagsets([[b"a"]])
    empty_q = tagsets([])
    with tmb.Database(one, keys=np.array([3], np.uint32)) as db:
        q, k = db.match_batch(empty_q, False)
        assert q.size == 0
        q, k = db.match_batch(tagsets([[b"a", b"b"], [b"b"]]), False)
        assert q.tolist() == [0] and k.tolist() == [3]
    with tmb.Database(tagsets([]), key_off=np.zeros(1, np.uint64), keys=np.zeros(0, np.uint32)) as db:
        q, k = db.match_batch(tagsets([[b"a"]]), True)
        assert q.size == 0


@pytest.mark.parametrize("layout", [(0, 0), (1, 1)])
def test_degenerate_databases(layout):
    """Identical sets (one row, Alg. 1 finds no pivot: reading R7), all-empty
    sets (the zero partition), a single set, and one set per tile boundary."""
    rnd = random.Random(2)
    cases = {
        "identical": [[b"a", b"b"]] * 1000,
        "all-empty": [[]] * 77,
        "single": [[b"x"]],
        "mixed-identical": [[b"a"]] * 500 + [[b"b"]] * 500 + [[]] * 3,
        "tile-ragged": [[f"t{rnd.randrange(9)}".encode() for _ in range(rnd.randint(1, 3))] for _ in range(33)],
    }
    queries = [[b"a", b"b"], [b"a"], [b"b", b"x"], [], [b"t1", b"t2", b"t3", b"a", b"x"]]
    for name, sets in cases.items():
        keys = [[i % 7, 1000 + i] for i in range(len(sets))]
        key_off = np.zeros(len(keys) + 1, np.uint64)
        key_off[1:] = np.cumsum([len(k) for k in keys])
        flat = np.array([k for kl in keys for k in kl], np.uint32)
        for max_p in (0xFFFFFFFF, 200_000, 10, 1):
            for unique in (False, True):
                want = o1.match([o1.encode(x) for x in sets], keys, [o1.encode(q) for q in queries], unique)
                with tmb.Database(tagsets(sets), key_off, flat, max_partition=max_p, tile_filter=layout[0],
                                  row_order=layout[1]) as db:
                    gq, gk = db.match_batch(tagsets(queries), unique)
                assert list(zip(gq.tolist(), gk.tolist())) == want, (name, max_p, unique)


def test_range_errors():
    """Sizes beyond the u32 query / key space are rejected (TM_ERANGE)."""
    import ctypes
    from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tm
    ts = tm.HostTagSets(np.zeros(0, np.uint8), np.zeros(1, np.uint64), None, np.zeros(2, np.uint64))
    ts.c.n_sets = 1 << 32
    h = ctypes.c_void_p()
    assert tm.load().tm_build(ctypes.byref(ts.c), None, None, None, ctypes.byref(h)) == -5


def test_output_overflow_retry():
    """More pairs than the initial capacity: the library re-runs the scan."""
    sets = [[]] * 3 + [[f"t{i}".encode()] for i in range(100)]
    keys = [list(range(1500))] * 3 + [[i] for i in range(100)]   # > 64 * 4500 pairs > initial capacity
    key_off = np.zeros(len(keys) + 1, np.uint64)
    key_off[1:] = np.cumsum([len(k) for k in keys])
    flat = np.array([k for kl in keys for k in kl], np.uint32)
    queries = [[f"t{i}".encode() for i in range(j, j + 40)] for j in range(64)]
    want = o1.match([o1.encode(s) for s in sets], keys, [o1.encode(q) for q in queries], False)
    with tmb.Database(tagsets(sets), key_off, flat, max_partition=20) as db:
        gq, gk = db.match_batch(tagsets(queries), False)
        assert db.stats()["retries"] >= 1
    assert list(zip(gq.tolist(), gk.tolist())) == want


class _CAI:
    """Expose a device pointer through __cuda_array_interface__ (torch.as_tensor reads it)."""

    def __init__(self, ptr, n, typestr="<u4"):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}


def _malformed_batches(c1):
    """(what, TagSets) query batches whose CSR breaks include/tagmatch.h's rules in the middle
    (the O(1) end-point checks pass; only the encoder kernels' device validation sees it)."""
    q = c1.queries
    vo, ti, so = q.vocab_off.copy(), q.tag_idx.copy(), q.set_off.copy()
    bad_so = so.copy()
    bad_so[5], bad_so[6] = so[6], so[5]                      # non-decreasing broken
    bad_ti = ti.copy()
    bad_ti[17] = q.vocab_off.size + 1000                     # index past the vocabulary
    bad_vo = vo.copy()
    bad_vo[3] = vo[-1] + 7                                   # string past n_bytes
    return [("set_off", tmgen.TagSets(q.vocab_bytes, vo, ti, bad_so)),
            ("tag_idx", tmgen.TagSets(q.vocab_bytes, vo, bad_ti, so)),
            ("vocab_off", tmgen.TagSets(q.vocab_bytes, bad_vo, ti, so))]


def test_malformed_query_batch_is_rejected(c1):
    """A malformed query CSR fails with TM_EINVAL on both entry points (validated on the device by
    the encoder, no out-of-bounds read), and the handle keeps working afterwards."""
    torch = pytest.importorskip("torch")
    want = oracle_pairs(c1, False)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=2000, tile_filter=1, row_order=1) as db:
        for what, bad in _malformed_batches(c1):
            with pytest.raises(tmb.TagMatchError) as e:
                db.match_batch(bad, False)
            assert e.value.status == -1, what
            t = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in
                 (bad.vocab_bytes, bad.vocab_off.view(np.int64), bad.tag_idx.view(np.int32),
                  bad.set_off.view(np.int64))]
            dq = tmb.device_tagsets(t[0].data_ptr(), t[1].data_ptr(), t[2].data_ptr(), t[3].data_ptr(),
                                    bad.vocab_bytes.size, bad.vocab_off.size - 1, bad.tag_idx.size, bad.n_sets)
            with pytest.raises(tmb.TagMatchError) as e:
                db.match_batch_device(dq, False, torch.cuda.current_stream().cuda_stream)
            assert e.value.status == -1, what
            assert_pairs_equal(db.match_batch(c1.queries, False), want, f"after malformed {what}")


def test_variant_tuning_flag(c1, c2, c2_oracle, monkeypatch):
    """tm_stats.tuning: 1 while the handle still times variants for this batch size (it then
    cycles through them), 0 once it has settled; never set for forced variants or streaming calls."""
    monkeypatch.delenv("TM_SCAN_VARIANT", raising=False)
    want = c2_oracle[False]
    with tmb.Database(c2.db, c2.key_off, c2.keys, max_partition=c2.max_partition, tile_filter=1,
                      row_order=1) as db:
        flags, variants = [], []
        for _ in range(10):
            assert_pairs_equal(db.match_batch(c2.queries, False), want, "during tuning")
            st = db.stats()
            flags.append(st["tuning"])
            variants.append(st["scan_variant"])
        assert flags[0] == 1 and 0 in flags, flags
        settled = flags.index(0)
        assert all(f == 0 for f in flags[settled:]) and len(set(variants[settled + 1:])) == 1, (flags, variants)
        assert {14, 8} <= set(variants[:settled + 1]), variants   # kTune (tm_internal.h)
        db.match_batch(c2.queries.subset(np.arange(3)), False)    # streaming-only call
        assert db.stats()["tuning"] == 0
    monkeypatch.setenv("TM_SCAN_VARIANT", "5")
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=2000, tile_filter=1, row_order=1) as db:
        db.match_batch(c1.queries, False)
        assert db.stats()["tuning"] == 0


@pytest.mark.parametrize("unique", [False, True])
def test_csr_result_equals_pairs(c1, unique):
    """tm_match_batch_csr returns the pairs of tm_match_batch as per-query key lists, also for
    queries without matches and for an empty batch."""
    extra = tagsets([[b"zz-none-1"], [], [b"zz-none-2", b"zz-none-3"]])
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=2000, tile_filter=1, row_order=1) as db:
        for qs in (c1.queries, extra, c1.queries.subset(np.arange(0))):
            q, k = db.match_batch(qs, unique)
            off, key = db.match_batch_csr(qs, unique)
            Q = qs.n_sets
            assert off.size == Q + 1 and off[0] == 0 and off[-1] == key.size
            assert np.all(np.diff(off.astype(np.int64)) >= 0)
            assert np.array_equal(np.repeat(np.arange(Q, dtype=np.uint32), np.diff(off).astype(np.int64)), q)
            assert np.array_equal(key, k)


def test_device_entry_point_matches_host(c1):
    torch = pytest.importorskip("torch")
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=200_000) as db:
        for unique in (False, True):
            hq, hk = db.match_batch(c1.queries, unique)
            t = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in
                 (c1.queries.vocab_bytes, c1.queries.vocab_off.view(np.int64), c1.queries.tag_idx.view(np.int32),
                  c1.queries.set_off.view(np.int64))]
            dq = tmb.device_tagsets(t[0].data_ptr(), t[1].data_ptr(), t[2].data_ptr(), t[3].data_ptr(),
                                    c1.queries.vocab_bytes.size, c1.queries.vocab_off.size - 1,
                                    c1.queries.tag_idx.size, c1.queries.n_sets)
            stream = torch.cuda.current_stream().cuda_stream
            out = db.match_batch_device(dq, unique, stream)
            gq = torch.as_tensor(_CAI(out.query, out.n), device="cuda").cpu().numpy().view(np.uint32)
            gk = torch.as_tensor(_CAI(out.key, out.n), device="cuda").cpu().numpy().view(np.uint32)
            assert_pairs_equal((gq, gk), (hq, hk), f"device API unique={unique}")


# ------------------------------------------------------------- streaming --
@pytest.mark.parametrize("max_batch,timeout_us", [(64, 200), (1_000_000, 500), (7, 0)])
def test_stream_one_query_at_a_time(c1, max_batch, timeout_us):
    """tm_stream: one-query submissions, batches closed by size or
    timeout; every query's keys equal the oracle's."""
    from paper_conf_eurosys_rogorapkmcc17_b200.tagmatch import Stream
    want_q, want_k = oracle_pairs(c1, True)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=200_000) as db:
        with Stream(db, max_batch, timeout_us, unique=True) as st:
            tickets = [st.submit(c1.queries.strings(j)) for j in range(300)]
            st.flush()
            got = {}
            while True:
                r = st.poll(wait=False)
                if r is None:
                    break
                assert r["n_queries"] if "n_queries" in r else True
                for i, t in enumerate(r["tickets"]):
                    got[int(t)] = r["keys"][r["key_off"][i]:r["key_off"][i + 1]]
                assert r["done_ns"] >= r["dispatch_ns"] >= r["submit_ns"].max()
                if max_batch < 300:
                    assert r["tickets"].size <= max_batch
    assert sorted(got) == tickets
    for j in range(300):
        assert np.array_equal(got[j], want_k[want_q == j])


def test_stream_replay_open_loop(c1):
    from paper_conf_eurosys_rogorapkmcc17_b200.tagmatch import Stream
    want_q, want_k = oracle_pairs(c1, False)
    arrivals = np.cumsum(np.random.default_rng(3).exponential(20_000, c1.queries.n_sets)).astype(np.uint64)
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=200_000) as db:
        with Stream(db, 128, 1000, unique=False) as st:
            st.replay(c1.queries, arrivals)
            st.flush()
            got = {}
            while (r := st.poll(wait=False)) is not None:
                for i, t in enumerate(r["tickets"]):
                    got[int(t)] = r["keys"][r["key_off"][i]:r["key_off"][i + 1]]
    assert sorted(got) == list(range(c1.queries.n_sets))
    for j in range(c1.queries.n_sets):
        assert np.array_equal(got[j], want_k[want_q == j])


# ------------------------------------------------------------ exact mode --
def _exact_oracle(db_strings, key_lists, q_strings, unique, db_sig, q_sig):
    """Exact containment on strings, evaluated on the Bloom candidates only
    (sound: exact containment implies Bloom containment, pinned in
    tests/test_oracle_pins.py)."""
    sets = [frozenset(s) for s in db_strings]
    out = []
    for j in range(len(q_strings)):
        qs = frozenset(q_strings[j])
        cand = np.nonzero(((db_sig[:, 0] & ~q_sig[j, 0]) | (db_sig[:, 1] & ~q_sig[j, 1]) |
                           (db_sig[:, 2] & ~q_sig[j, 2])) == 0)[0]
        ks = [k for i in cand if sets[i] <= qs for k in key_lists[i]]
        ks = sorted(set(ks)) if unique else sorted(ks)
        out.extend((j, k) for k in ks)
    return out


@pytest.mark.parametrize("unique", [False, True])
def test_exact_mode_removes_false_positives(unique):
    """Dense queries over a 50-tag vocabulary produce many Bloom false
    positives; exact mode returns exactly the string-level containment."""
    rnd = random.Random(8)
    vocab = [f"w{i}".encode() for i in range(50)] + [b"", b"\x00\xff"]
    sets = [[rnd.choice(vocab) for _ in range(rnd.randint(0, 4))] for _ in range(3000)]
    sets += [[b"w1", b"w1"], [b"w2", b"w1"]]
    keys = [[rnd.randrange(1000) for _ in range(rnd.randint(0, 2))] for _ in range(len(sets))]
    queries = [[rnd.choice(vocab) for _ in range(rnd.randint(10, 40))] for _ in range(200)]
    queries += [[], [b"zz"], vocab]
    key_off = np.zeros(len(keys) + 1, np.uint64)
    key_off[1:] = np.cumsum([len(k) for k in keys])
    flat = np.array([k for kl in keys for k in kl], np.uint32)
    want = o1.match_exact(sets, keys, queries, unique)
    bloom = o1.match([o1.encode(s) for s in sets], keys, [o1.encode(q) for q in queries], unique)
    assert len(bloom) > len(want)          # the workload does have false positives
    for max_p in (0xFFFFFFFF, 100, 1):
        with tmb.Database(tagsets(sets), key_off, flat, max_partition=max_p, exact=1) as db:
            gq, gk = db.match_batch(tagsets(queries), unique)
            st = db.stats()
        assert list(zip(gq.tolist(), gk.tolist())) == want
        assert st["exact_kept"] <= st["exact_checked"]


def test_exact_mode_duplicate_vocabulary_strings():
    """Vocabulary entries with identical bytes are one tag (canonical ids)."""
    vb = np.frombuffer(b"aabbaa", np.uint8)
    vo = np.array([0, 2, 4, 6], np.uint64)            # "aa", "bb", "aa"
    db_ts = tmgen.TagSets(vb, vo, np.array([0, 1, 2], np.uint32), np.array([0, 2, 3], np.uint64))
    q_ts = tagsets([[b"aa", b"bb"], [b"aa"], [b"bb"]])
    with tmb.Database(db_ts, keys=np.array([5, 6], np.uint32), exact=1) as db:
        q, k = db.match_batch(q_ts, False)
    assert list(zip(q.tolist(), k.tolist())) == [(0, 5), (0, 6), (1, 6)]


@pytest.mark.parametrize("unique", [False, True])
def test_exact_mode_c1(c1, unique):
    db_strings = [c1.db.strings(i) for i in range(c1.db.n_sets)]
    q_strings = [c1.queries.strings(j) for j in range(c1.queries.n_sets)]
    key_lists = [c1.keys[c1.key_off[i]:c1.key_off[i + 1]].tolist() for i in range(c1.db.n_sets)]
    want = _exact_oracle(db_strings, key_lists, q_strings, unique, o2.encode(c1.db), o2.encode(c1.queries))
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=500, tile_filter=1, row_order=1, exact=1) as db:
        gq, gk = db.match_batch(c1.queries, unique)
    assert list(zip(gq.tolist(), gk.tolist())) == want


def test_exact_mode_c2_sample(c2):
    """Exact mode at C2 size on a 300-query sample: string-level containment."""
    rng = np.random.default_rng(5)
    qsel = np.sort(rng.choice(c2.queries.n_sets, 300, replace=False))
    db_sig, q_sig = o2.encode(c2.db), o2.encode(c2.queries)
    want = []
    for j in qsel:
        qs = frozenset(c2.queries.strings(int(j)))
        cand = np.nonzero(((db_sig[:, 0] & ~q_sig[j, 0]) | (db_sig[:, 1] & ~q_sig[j, 1]) |
                           (db_sig[:, 2] & ~q_sig[j, 2])) == 0)[0]
        ks = sorted(k for i in cand if frozenset(c2.db.strings(int(i))) <= qs
                    for k in c2.keys[c2.key_off[i]:c2.key_off[i + 1]].tolist())
        want.extend((int(j), k) for k in ks)
    with tmb.Database(c2.db, c2.key_off, c2.keys, max_partition=c2.max_partition, tile_filter=1, row_order=1,
                      exact=1) as db:
        gq, gk = db.match_batch(c2.queries, False)
    keep = np.isin(gq, qsel)
    assert list(zip(gq[keep].tolist(), gk[keep].tolist())) == want


# ------------------------------------------ sec. 4.4 crafted workload (C6/C7 shapes) --
@pytest.mark.parametrize("s,t", [(2, 10), (3, 6)])
@pytest.mark.parametrize("unique", [False, True])
def test_crafted_workload_parity(s, t, unique):
    """The sec. 4.4 workload at a size the brute-force oracle finishes in
    seconds: 300K sets of s tags, 4,000 queries of t tags; bit-exact vs O2 brute force; every
    query returns its base set's key (keys = set index)."""
    wl = tmgen.generate_crafted(300_000, s, t, 4000, seed=40 + s, max_partition=20_000)
    want = oracle_pairs(wl, unique)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition) as db:
        got = db.match_batch(wl.queries, unique)
    assert_pairs_equal(got, want, f"crafted s={s} t={t}")
    pairs = set(zip(got[0].tolist(), got[1].tolist()))
    assert all((j, int(b)) in pairs for j, b in enumerate(wl.query_base))


@pytest.mark.parametrize("s,t", [(2, 10), (3, 6)])
def test_crafted_workload_exact_mode(s, t):
    """Exact mode on the crafted workload: string-level containment, checked on a 300-query
    sample against the definition (the Bloom candidates of O2, then exact set containment)."""
    wl = tmgen.generate_crafted(300_000, s, t, 2000, seed=50 + s)
    rng = np.random.default_rng(6)
    qsel = np.sort(rng.choice(wl.queries.n_sets, 300, replace=False))
    db_sig, q_sig = o2.encode(wl.db), o2.encode(wl.queries)
    want = []
    for j in qsel:
        qs = frozenset(wl.queries.strings(int(j)))
        cand = np.nonzero(((db_sig[:, 0] & ~q_sig[j, 0]) | (db_sig[:, 1] & ~q_sig[j, 1]) |
                           (db_sig[:, 2] & ~q_sig[j, 2])) == 0)[0]
        want.extend((int(j), int(i)) for i in cand if frozenset(wl.db.strings(int(i))) <= qs)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, exact=1) as db:
        gq, gk = db.match_batch(wl.queries, False)
    keep = np.isin(gq, qsel)
    assert list(zip(gq[keep].tolist(), gk[keep].tolist())) == want


@pytest.mark.parametrize("ranges", ["1", "2", "3", "7"])
def test_csr_pipelined_ranges(c2, c2_oracle, ranges, monkeypatch):
    """Pipelined tm_match_batch_csr and tm_match_batch (TM_PIPELINE query ranges: the D2H of range k overlaps the
    GPU work of range k + 1; double-buffered keys, per-range query offsets): the per-query key
    lists equal the oracle's pairs for any number of ranges, uneven ones included, and the call's
    statistics are the sums over its ranges."""
    monkeypatch.setenv("TM_PIPELINE", ranges)
    with tmb.Database(c2.db, c2.key_off, c2.keys, max_partition=c2.max_partition, tile_filter=1,
                      row_order=1) as db:
        for unique in (False, True):
            for _ in range(2):   # the second call reuses the copy stream, buffers and pinned blocks
                off, key = db.match_batch_csr(c2.queries, unique)
                wq, wk = c2_oracle[unique]
                Q = c2.queries.n_sets
                assert off.size == Q + 1 and off[0] == 0 and off[-1] == key.size == wk.size
                assert np.array_equal(np.repeat(np.arange(Q, dtype=np.uint32), np.diff(off).astype(np.int64)), wq)
                assert np.array_equal(key, wk)
                st = db.stats()
                assert st["result_pairs"] == wk.size and st["n_queries"] == Q
                assert_pairs_equal(db.match_batch(c2.queries, unique), (wq, wk), f"pairs, {ranges} ranges")


def test_csr_pipelined_exact(monkeypatch):
    """The pipelined CSR call in exact mode (each query range runs the exact post-check) equals
    the oracle's string-level containment on a workload with many Bloom false positives."""
    monkeypatch.setenv("TM_PIPELINE", "3")
    rnd = random.Random(9)
    vocab = [f"w{i}".encode() for i in range(50)]
    sets = [[rnd.choice(vocab) for _ in range(rnd.randint(0, 4))] for _ in range(2000)]
    keys = [[rnd.randrange(1000) for _ in range(rnd.randint(0, 2))] for _ in range(len(sets))]
    queries = [[rnd.choice(vocab) for _ in range(rnd.randint(8, 30))] for _ in range(301)]
    key_off = np.zeros(len(keys) + 1, np.uint64)
    key_off[1:] = np.cumsum([len(k) for k in keys])
    flat = np.array([k for kl in keys for k in kl], np.uint32)
    for unique in (False, True):
        want = o1.match_exact(sets, keys, queries, unique)
        with tmb.Database(tagsets(sets), key_off, flat, max_partition=100, exact=1) as db:
            off, key = db.match_batch_csr(tagsets(queries), unique)
        q = np.repeat(np.arange(len(queries), dtype=np.uint32), np.diff(off).astype(np.int64))
        assert list(zip(q.tolist(), key.tolist())) == want
