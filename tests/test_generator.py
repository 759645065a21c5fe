"""The seeded workload generator: determinism and the paper's workload shape
(PAPER.md:262-282).  CPU only."""
import numpy as np

import tmgen
from oracle import o1, o2


def test_deterministic_and_thread_independent():
    a = tmgen.generate(3000, 200, seed=9, nthreads=1, keep_ids=True)
    b = tmgen.generate(3000, 200, seed=9, nthreads=5, keep_ids=True)
    for x, y in [(a.db_ids, b.db_ids), (a.db.set_off, b.db.set_off), (a.keys, b.keys),
                 (a.key_off, b.key_off), (a.q_ids, b.q_ids), (a.query_base, b.query_base)]:
        assert np.array_equal(x, y)
    c = tmgen.generate(3000, 200, seed=10, keep_ids=True)
    assert not np.array_equal(a.db_ids[:100], c.db_ids[:100])


def test_workload_shape(c1):
    lens = np.diff(c1.db.set_off)
    assert 4.8 < lens.mean() < 5.3                     # ~5 tags per interest
    assert lens.min() >= 1 and lens.max() <= 20
    kpl = np.diff(c1.key_off)
    assert 1.35 < kpl.mean() < 1.48                    # 300M keys / 212M sets
    ql = np.diff(c1.queries.set_off)
    # query = base set + 2..4 extra tags
    extra = ql - lens[c1.query_base.astype(np.int64)]
    assert extra.min() >= 2 and extra.max() <= 4


def test_db_sets_unique_and_queries_contain_base():
    w = tmgen.generate(20000, 500, seed=4, keep_ids=True)
    canon = {tuple(w.db_ids[w.db.set_off[i]:w.db.set_off[i + 1]]) for i in range(w.db.n_sets)}
    assert len(canon) == w.db.n_sets                    # unique sets
    for j in range(w.queries.n_sets):
        b = int(w.query_base[j])
        base = set(w.db_ids[w.db.set_off[b]:w.db.set_off[b + 1]].tolist())
        q = set(w.q_ids[w.queries.set_off[j]:w.queries.set_off[j + 1]].tolist())
        assert base <= q


def test_total_tags_sweep_mode():
    for t in (2, 6, 12):
        w = tmgen.generate(5000, 300, seed=500 + t, total_tags=t)
        assert np.all(np.diff(w.queries.set_off) == t)


def test_every_query_matches_its_base(c1):
    """Workload guarantee: each query matches >= 1 DB set."""
    db = o2.encode(c1.db)
    qs = o2.encode(c1.queries)
    base = db[c1.query_base.astype(np.int64)]
    assert np.all((base & ~qs) == 0)


def test_c1_oracles_agree(c1):
    """O1 (Python definition, numpy scan) == O2 brute == O2 partitioned on C1."""
    db = o2.encode(c1.db)
    qs = o2.encode(c1.queries)
    # O1 encoder on a sample of sets agrees with O2's
    for i in range(0, c1.db.n_sets, 997):
        assert o1.words(o1.encode(c1.db.strings(i))) == tuple(int(x) for x in db[i])
    for unique in (False, True):
        q1, k1 = o1.match_numpy(db, c1.key_off, c1.keys, qs[:200], unique)
        q2, k2 = o2.match_brute(db, c1.key_off, c1.keys, qs[:200], unique)
        assert np.array_equal(q1, q2) and np.array_equal(k1, k2)
        qa, ka = o2.match_brute(db, c1.key_off, c1.keys, qs, unique)
        for mp in (0xFFFFFFFF, 200_000, 1000):
            qb, kb, _ = o2.Index(db, mp).match(c1.key_off, c1.keys, qs, unique)
            assert np.array_equal(qa, qb) and np.array_equal(ka, kb)


def test_crafted_workload_shape():
    """Sec. 4.4 crafted workload: sets of exactly s distinct tags, distinct
    sets, queries of exactly t distinct tags that contain their base set; deterministic."""
    for s, t in ((2, 10), (3, 6)):
        w = tmgen.generate_crafted(20000, s, t, 500, seed=11)
        assert np.all(np.diff(w.db.set_off) == s) and np.all(np.diff(w.queries.set_off) == t)
        vb = w.db.vocab_bytes.tobytes()
        dstr = [vb[w.db.vocab_off[i]:w.db.vocab_off[i + 1]] for i in range(w.db.vocab_off.size - 1)]
        qb = w.queries.vocab_bytes.tobytes()
        qstr = [qb[w.queries.vocab_off[i]:w.queries.vocab_off[i + 1]] for i in range(w.queries.vocab_off.size - 1)]
        rows = [frozenset(dstr[x] for x in w.db.tag_idx[i * s:(i + 1) * s]) for i in range(w.db.n_sets)]
        assert all(len(r) == s for r in rows) and len(set(rows)) == w.db.n_sets
        for j in range(w.queries.n_sets):
            q = frozenset(qstr[x] for x in w.queries.tag_idx[j * t:(j + 1) * t])
            assert len(q) == t and rows[int(w.query_base[j])] <= q
        assert np.array_equal(w.keys, np.arange(w.db.n_sets, dtype=np.uint32))
        w2 = tmgen.generate_crafted(20000, s, t, 500, seed=11)
        assert np.array_equal(w.db.tag_idx, w2.db.tag_idx) and np.array_equal(w.queries.tag_idx, w2.queries.tag_idx)
