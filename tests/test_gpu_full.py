"""Parity at BASELINE.json's full sizes (C3: 100M tag sets x 1M queries; C4:
300M x 1M) in the configuration bench.py times, checked on a seeded sample of
queries that the oracle (O2, brute force over the whole database) computes
one by one.  Plus size-independent properties of the whole output.

C3 runs by default (about 2 minutes on a B200: generation 25 s, GPU build 3 s,
oracle samples 10 s); `TM_FULL_SIZE=C4` selects C4, `TM_FULL_SIZE=0` skips.
"""
import os
import time

import numpy as np
import pytest

import tmgen
from oracle import o2

pytestmark = [pytest.mark.gpu, pytest.mark.slow,
              pytest.mark.skipif(os.environ.get("TM_FULL_SIZE", "C3") == "0", reason="TM_FULL_SIZE=0")]
tmb = pytest.importorskip("paper_conf_eurosys_rogorapkmcc17_b200")


@pytest.fixture(scope="module")
def full():
    name = os.environ.get("TM_FULL_SIZE", "C3")
    name = name if name in tmgen.CONFIGS else "C3"
    t = time.time()
    wl = tmgen.config(name)
    print(f"\n{name}: generated {wl.db.n_sets} sets, {wl.queries.n_sets} queries in {time.time() - t:.1f} s")
    t = time.time()
    # the layout bench.py times by default: balanced splits + tile AND masks (R18)
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1, row_order=1)
    st = db.stats()
    print(f"{name}: built in {time.time() - t:.1f} s: {st['n_partitions']} partitions, {st['n_unique']} rows")
    yield name, wl, db
    db.close()


@pytest.mark.parametrize("unique", [False, True])
def test_full_size_sampled_parity(full, unique):
    name, wl, db = full
    t = time.time()
    gq, gk = db.match_batch(wl.queries, unique)
    st = db.stats()
    print(f"{name} unique={unique}: {gq.size} pairs in {time.time() - t:.2f} s (scan {st['scan_ms']:.1f} ms, "
          f"{st['candidate_pairs']:.3e} candidate pairs, {st['pair_checks']:.3e} checks)")
    # properties of the whole output: sorted, query ids in range, every query matches its base
    key = (gq.astype(np.uint64) << np.uint64(32)) | gk.astype(np.uint64)
    assert np.all(key[1:] >= key[:-1])
    if unique:
        assert np.all(key[1:] != key[:-1])
    assert gq.size == 0 or gq.max() < wl.queries.n_sets
    assert np.unique(gq).size == wl.queries.n_sets
    # sampled bit-exact parity against brute force over the whole database
    rng = np.random.default_rng(2024 + unique)
    qsel = np.sort(rng.choice(wl.queries.n_sets, 192, replace=False))
    t = time.time()
    db_sig = o2.encode(wl.db)
    qs = o2.encode(wl.queries.subset(qsel))
    wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, qs, unique, qid=qsel.astype(np.uint32))
    print(f"oracle sample: {time.time() - t:.1f} s")
    keep = np.isin(gq, qsel)
    assert np.array_equal(gq[keep], wq) and np.array_equal(gk[keep], wk)


@pytest.mark.parametrize("name", ["C6", "C7"])
def test_crafted_full_size_sampled_parity(name):
    """The sec. 4.4 crafted workloads at full size (C6: 5M 2-tag sets x 100k 10-tag queries;
    C7: 3M x 3 tags x 100k 6-tag queries) in the layout bench.py times:
    whole-output properties, then bit-exact parity on a 192-query sample against O2 brute force
    over the whole database, for match and match-unique."""
    wl = tmgen.config(name)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, tile_filter=1,
                      row_order=1) as db:
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
            qs = o2.encode(wl.queries.subset(qsel))
            wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, qs, unique, qid=qsel.astype(np.uint32))
            keep = np.isin(gq, qsel)
            assert np.array_equal(gq[keep], wq) and np.array_equal(gk[keep], wk)
