"""Seeded randomized parity: random small databases and batches through every
combination of the library's options (MAX_P, pre-filter, row order, exact
check, match / match-unique, scan-kernel variant), compared with the oracle's
definition (o1.match on signatures, o1.match_exact on strings)."""
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


@pytest.mark.parametrize("case", range(40))
def test_random_configuration(case, monkeypatch):
    rnd = random.Random(1000 + case)
    nv = rnd.randint(3, 90)
    vocab = [f"v{i}".encode() for i in range(nv)] + ([b""] if rnd.random() < 0.3 else [])
    n_sets = rnd.choice([0, 1, 5, 31, 32, 33, 200, 1500, 4000])
    sets = [[rnd.choice(vocab) for _ in range(rnd.randint(0, 8))] for _ in range(n_sets)]
    keys = [[rnd.randrange(64) for _ in range(rnd.randint(0, 3))] for _ in range(n_sets)]
    n_q = rnd.choice([0, 1, 3, 8, 9, 40, 300])
    queries = [[rnd.choice(vocab) for _ in range(rnd.randint(0, 30))] for _ in range(n_q)]
    max_p = rnd.choice([1, 3, 17, 200, 0xFFFFFFFF])
    tile_filter = rnd.choice([0, 1, 2])
    row_order = rnd.choice([0, 1]) if tile_filter else 0
    exact = rnd.random() < 0.35
    unique = rnd.random() < 0.5
    variant = rnd.choice(["", "0", "5", "5", "6", "7", "8", "9", "10", "11", "12", "13", "14", "14", "15", "16", "17", "17", "18"])
    if variant:
        monkeypatch.setenv("TM_SCAN_VARIANT", variant)
    else:
        monkeypatch.delenv("TM_SCAN_VARIANT", raising=False)
    if exact:
        want = o1.match_exact(sets, keys, queries, unique)
    else:
        want = o1.match([o1.encode(s) for s in sets], keys, [o1.encode(q) for q in queries], unique)
    key_off = np.zeros(n_sets + 1, np.uint64)
    if n_sets:
        key_off[1:] = np.cumsum([len(k) for k in keys])
    flat = np.array([k for kl in keys for k in kl], np.uint32)
    with tmb.Database(_tagsets(sets), key_off, flat, max_partition=max_p, tile_filter=tile_filter,
                      row_order=row_order, exact=int(exact)) as db:
        for _ in range(2):   # second call: reused buffers, tuned variant
            gq, gk = db.match_batch(_tagsets(queries), unique)
            assert list(zip(gq.tolist(), gk.tolist())) == want, dict(
                case=case, n_sets=n_sets, n_q=n_q, max_p=max_p, tile_filter=tile_filter, row_order=row_order,
                exact=exact, unique=unique, variant=variant)
