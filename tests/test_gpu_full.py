"""Parity at BASELINE.json's full sizes in the configuration bench.py times (auto MAX_P; C3 / C4
also at the paper's 200K, whose whole output must be identical), checked on
seeded samples of queries that the oracle (O2, brute force over the WHOLE database, no
partitioning or pre-filter: the plain definition of SURVEY 8(c)) computes one by one, plus
size-independent properties of the whole output:

  C3  100M tag sets x 1M queries            2,048-query sample   (PAPER.md:262 scale, Fig. 4)
  C4  300M tag sets x 1M queries            512-query sample     (300M keys)
  C5  100M tag sets, t = 2 / 8 / 20 tags    256-query sample per t

All run by default (about 6 minutes on a B200: generation dominates); TM_FULL_SIZE=0 skips,
TM_FULL_SIZE=C3 (or C4, C5) runs one of them.
"""
import gc
import os
import time

import numpy as np
import pytest

import tmgen
from oracle import o2

_SEL = os.environ.get("TM_FULL_SIZE", "all")
pytestmark = [pytest.mark.gpu, pytest.mark.slow, pytest.mark.skipif(_SEL == "0", reason="TM_FULL_SIZE=0")]
tmb = pytest.importorskip("paper_conf_eurosys_rogorapkmcc17_b200")

SAMPLE = {"C3": 2048, "C4": 512}
C5_TOTALS = (2, 8, 20)
C5_SAMPLE = 256


def _want(name):
    return _SEL in ("all", "1", name)


def _sorted_props(gq, gk, n_queries, unique):
    key = (gq.astype(np.uint64) << np.uint64(32)) | gk.astype(np.uint64)
    assert np.all(key[1:] > key[:-1]) if unique else np.all(key[1:] >= key[:-1])
    assert gq.size == 0 or gq.max() < n_queries


def _sample_parity(db_sig, wl_key_off, wl_keys, queries, gq, gk, qsel, unique):
    """Bit-exact: the library's pairs of the sampled queries == O2 brute force over the whole DB."""
    qs = o2.encode(queries.subset(qsel))
    wq, wk = o2.match_brute(db_sig, wl_key_off, wl_keys, qs, unique, qid=qsel.astype(np.uint32))
    keep = np.isin(gq, qsel)
    assert np.array_equal(gq[keep], wq), f"query ids differ: {gq[keep].size} vs {wq.size} pairs"
    assert np.array_equal(gk[keep], wk), "keys differ"
    return wq.size


@pytest.fixture(scope="module", params=["C3", "C4"])
def full(request):
    name = request.param
    if not _want(name):
        pytest.skip(f"TM_FULL_SIZE={_SEL}")
    t = time.time()
    wl = tmgen.config(name)
    print(f"\n{name}: generated {wl.db.n_sets} sets, {wl.queries.n_sets} queries in {time.time() - t:.1f} s")
    dbs = []
    # the layout bench.py times by default: balanced splits + tile AND masks (R18), at the
    # MAX_P bench.py uses (TM_AUTO_MAX_PARTITION: 5K at C3, 10K at C4) and at the paper's 200K
    for mp in (tmb.TM_AUTO_MAX_PARTITION, wl.max_partition):
        t = time.time()
        db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp, tile_filter=1, row_order=1)
        st = db.stats()
        print(f"{name}: built in {time.time() - t:.1f} s: {st['n_partitions']} partitions, {st['n_unique']} rows")
        dbs.append(db)
    db_sig = o2.encode(wl.db)
    yield name, wl, dbs, db_sig
    for db in dbs:
        db.close()
    del wl, db_sig
    gc.collect()


@pytest.mark.parametrize("unique", [False, True])
def test_full_size_sampled_parity(full, unique):
    name, wl, dbs, db_sig = full
    outs = []
    for db in dbs:
        t = time.time()
        gq, gk = db.match_batch(wl.queries, unique)
        st = db.stats()
        print(f"{name} unique={unique} ({st['n_partitions']} partitions): {gq.size} pairs in {time.time() - t:.2f} s "
              f"(scan {st['scan_ms']:.1f} ms, {st['candidate_pairs']:.3e} candidate pairs, "
              f"{st['pair_checks']:.3e} checks)")
        # properties of the whole output: sorted, ids in range, every query matches its base
        _sorted_props(gq, gk, wl.queries.n_sets, unique)
        assert np.unique(gq).size == wl.queries.n_sets
        outs.append((gq, gk))
    # partitioning is lossless (Alg. 1 / Alg. 2): both MAX_P give the same whole output
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    # sampled bit-exact parity against brute force over the whole database
    rng = np.random.default_rng(2024 + unique + (10 if name == "C4" else 0))
    qsel = np.sort(rng.choice(wl.queries.n_sets, SAMPLE[name], replace=False))
    t = time.time()
    n = _sample_parity(db_sig, wl.key_off, wl.keys, wl.queries, outs[0][0], outs[0][1], qsel, unique)
    print(f"oracle sample of {qsel.size} queries ({n} pairs): {time.time() - t:.1f} s")


def test_c5_query_size_sweep_sampled_parity():
    """C5: one 100M-set database, query batches of t = 2, 8, 20 total tags
    (100k queries each); match and match-unique bit-exact on a 256-query sample per t, and the
    match rate grows with t (the paper's E2/E3 trend: more tags, more matches)."""
    if not _want("C5"):
        pytest.skip(f"TM_FULL_SIZE={_SEL}")
    t = time.time()
    wl, batches, bases = tmgen.generate_sweep(100_000_000, 500, 100_000, C5_TOTALS, 500)
    print(f"\nC5: generated in {time.time() - t:.1f} s")
    db_sig = o2.encode(wl.db)
    rates = []
    # the MAX_P of scripts/sweep_c5.py and bench.py (TM_AUTO_MAX_PARTITION: 5K at 100M sets)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=tmb.TM_AUTO_MAX_PARTITION, tile_filter=1,
                      row_order=1) as db:
        for tt in C5_TOTALS:
            q = batches[tt]
            for unique in (False, True):
                gq, gk = db.match_batch(q, unique)
                _sorted_props(gq, gk, q.n_sets, unique)
                rng = np.random.default_rng(500 + tt + unique)
                qsel = np.sort(rng.choice(q.n_sets, C5_SAMPLE, replace=False))
                n = _sample_parity(db_sig, wl.key_off, wl.keys, q, gq, gk, qsel, unique)
                if not unique:
                    rates.append(gq.size / q.n_sets)
                print(f"C5 t={tt} unique={unique}: {gq.size} pairs, sample {n} pairs ok")
    assert rates == sorted(rates), f"match rate must grow with query size: {rates}"


@pytest.mark.parametrize("name", ["C6", "C7"])
def test_crafted_full_size_sampled_parity(name):
    """The sec. 4.4 crafted workloads at full size (C6: 5M 2-tag sets x 100k 10-tag queries;
    C7: 3M x 3 tags x 100k 6-tag queries) in the layout bench.py times:
    whole-output properties, then bit-exact parity on a 192-query sample against O2 brute force
    over the whole database, for match and match-unique."""
    wl = tmgen.config(name)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=tmb.TM_AUTO_MAX_PARTITION, tile_filter=1,
                      row_order=1) as db:   # bench.py's MAX_P for these (auto)
        db_sig = o2.encode(wl.db)
        for unique in (False, True):
            gq, gk = db.match_batch(wl.queries, unique)
            key = (gq.astype(np.uint64) << np.uint64(32)) | gk.astype(np.uint64)
            assert np.all(key[1:] > key[:-1]) if unique else np.all(key[1:] >= key[:-1])
            # every query returns its base set's key (key = set index)
            base_key = (np.arange(wl.queries.n_sets, dtype=np.uint64) << np.uint64(32)) | wl.query_base
            assert np.all(np.isin(base_key, key))
            rng = np.random.default_rng(77 + unique)
            qsel = np.sort(rng.choice(wl.queries.n_sets, 192, replace=False))
            _sample_parity(db_sig, wl.key_off, wl.keys, wl.queries, gq, gk, qsel, unique)
