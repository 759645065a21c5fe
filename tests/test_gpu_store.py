"""add-set / remove-set / consolidate (Table 2; NEXT-3): seeded random sequences of
staged operations with consolidates in between, on a mutable handle (tm_create), compared after
every consolidate with the oracle's definition (o1.match on the live multiset of (set, key)
entries; o1.match_exact in exact mode).  Staged changes are invisible until consolidate; a
remove-set removes one instance of an identical entry (R20)."""
import random

import numpy as np
import pytest

import tmgen
from oracle import o1

pytestmark = pytest.mark.gpu
tmb = pytest.importorskip("paper_conf_eurosys_rogorapkmcc17_b200")


def _tagsets(strings_per_set):
    flat = [t for s in strings_per_set for t in s]
    vb = np.frombuffer(b"".join(flat), np.uint8) if any(flat) else np.zeros(0, np.uint8)
    vo = np.zeros(len(flat) + 1, np.uint64)
    if flat:
        vo[1:] = np.cumsum([len(t) for t in flat])
    so = np.zeros(len(strings_per_set) + 1, np.uint64)
    if strings_per_set:
        so[1:] = np.cumsum([len(s) for s in strings_per_set])
    return tmgen.TagSets(vb, vo, np.arange(len(flat), dtype=np.uint32), so)


def _want(live, queries, unique, exact):
    sets = [s for s, _ in live]
    keys = [[k] for _, k in live]
    if exact:
        return o1.match_exact(sets, keys, queries, unique)
    return o1.match([o1.encode(s) for s in sets], keys, [o1.encode(q) for q in queries], unique)


def _got(db, queries, unique):
    gq, gk = db.match_batch(_tagsets(queries), unique)
    return list(zip(gq.tolist(), gk.tolist()))


@pytest.mark.parametrize("case", range(6))
def test_staged_operations_match_oracle(case):
    rnd = random.Random(77 + case)
    vocab = [f"t{i}".encode() for i in range(rnd.randint(8, 60))]
    exact = case % 3 == 2
    n_gpus = 2 if case % 2 else 0
    kw = dict(max_partition=rnd.choice([3, 50, 0]), tile_filter=1, row_order=1, exact=int(exact))
    if n_gpus:
        kw.update(n_gpus=2, device_ids=[0, 0], shard_mode=case % 4 // 2)
    db = tmb.Database.create(**kw)
    queries = [[rnd.choice(vocab) for _ in range(rnd.randint(0, 14))] for _ in range(120)]
    live = []        # the consolidated multiset of (set, key) entries, as the oracle sees it
    staged = []
    try:
        assert _got(db, queries, False) == []   # empty before the first consolidate
        for rnd_i in range(4):
            for _ in range(rnd.randint(50, 400)):
                if live and rnd.random() < 0.3:   # remove an existing entry (its tags reordered, repeated)
                    s, k = rnd.choice(live + [e for op, e in staged if op])
                    t = list(s) + ([s[0]] if s and rnd.random() < 0.3 else [])
                    rnd.shuffle(t)
                    db.remove_set(t, k)
                    staged.append((False, (tuple(sorted(set(s))), k)))
                elif rnd.random() < 0.05:         # remove something that is not there
                    db.remove_set([b"absent"], 7)
                    staged.append((False, ((b"absent",), 7)))
                else:
                    s = [rnd.choice(vocab) for _ in range(rnd.randint(0, 6))]
                    k = rnd.randrange(40)
                    db.add_set(s, k)
                    staged.append((True, (tuple(sorted(set(s))), k)))
            # staged changes are not visible yet
            for unique in (False, True):
                assert _got(db, queries, unique) == _want(live, queries, unique, exact)
            n_staged, n_live = db.pending()
            assert n_staged == len(staged) and n_live == len(live)
            db.consolidate()
            for op, e in staged:   # apply in call order: remove one instance if present
                if op:
                    live.append(e)
                elif e in live:
                    live.remove(e)
            staged = []
            assert db.pending() == (0, len(live))
            for unique in (False, True):
                assert _got(db, queries, unique) == _want(live, queries, unique, exact), (case, rnd_i, unique)
    finally:
        db.close()


def test_bulk_add_sets_equals_build():
    """add_sets (add-set for every entry of a batch) + consolidate == tm_build of the same input."""
    wl = tmgen.generate(5000, 500, seed=9, max_partition=300)
    with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=300, tile_filter=1, row_order=1) as ref:
        want = ref.match_batch(wl.queries, False)
    db = tmb.Database.create(max_partition=300, tile_filter=1, row_order=1)
    try:
        db.add_sets(wl.db, wl.key_off, wl.keys)
        assert db.pending()[0] == int(wl.key_off[-1])
        db.consolidate()
        got = db.match_batch(wl.queries, False)
        assert np.array_equal(got[0], want[0]) and np.array_equal(got[1], want[1])
    finally:
        db.close()


def test_built_handle_is_not_mutable(c1):
    with tmb.Database(c1.db, c1.key_off, c1.keys, max_partition=500) as db:
        with pytest.raises(tmb.TagMatchError) as e:
            db.add_set([b"x"], 1)
        assert e.value.status == -6
