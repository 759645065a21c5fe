"""Pins of the ORACLE against things other than itself (CPU only).

Each test names what fixes the expected value: a published test vector, a
value the paper prints, a closed form, an invariant, or brute force on tiny
inputs.  See DESIGN.md "Oracle and its pins".
"""
import ast
import itertools
import math
import random

import numpy as np
import pytest

from conftest import golden_lines
from oracle import o1, o2


# ---------------------------------------------------------------- encoder ---
def test_fnv1a64_published_vectors():
    """FNV-1a-64 reference vectors (tests/golden/fnv1a64.txt); both oracles."""
    for line in golden_lines("fnv1a64.txt"):
        lit, hexd = line.rsplit(None, 1)
        data = ast.literal_eval(lit.strip())
        assert o1.fnv1a64(data) == int(hexd, 16)
        assert o2.fnv1a64(data) == int(hexd, 16)


def test_splitmix64_published_sequence():
    """SplitMix64 reference outputs for seed 1234567 (tests/golden/splitmix64.txt)."""
    lines = golden_lines("splitmix64.txt")
    state = int(lines[0].split()[1])
    for want in lines[1:]:
        state, z = o1.splitmix64(state)
        assert z == int(want)
    # O2's mix is the same output function applied to state + (r+1)*golden
    state = int(lines[0].split()[1])
    for r, want in enumerate(lines[1:]):
        assert o2.splitmix_mix((state + (r + 1) * o1.GOLDEN) % 2**64) == int(want)


def test_positions_are_lemire_reduction():
    """pos = floor(z * 192 / 2^64), i.e. the integer part of 192 * (z / 2^64);
    checked in exact rational arithmetic, independent of the >> form."""
    from fractions import Fraction
    for tag in [b"", b"cat", b"fr_cat", b"u123", b"en_t0"]:
        state = o1.fnv1a64(tag)
        pos = o1.tag_positions(tag)
        for r in range(7):
            state, z = o1.splitmix64(state)
            assert pos[r] == math.floor(Fraction(z, 2**64) * 192)
            assert 0 <= pos[r] < 192


def test_o1_o2_encoders_agree():
    """The two independently written oracle encoders give identical positions."""
    rnd = random.Random(7)
    tags = [b"", b"cat", b"fr_cat", b"u123"] + [bytes(rnd.getrandbits(8) for _ in range(rnd.randrange(0, 40)))
                                             for _ in range(500)]
    for t in tags:
        assert o1.tag_positions(t) == o2.tag_positions(t)


def test_bit_layout_msb_first():
    """Reading R3: position p in word p>>6 at bit 63-(p&63)."""
    for p in [0, 1, 63, 64, 127, 128, 191]:
        w = o1.words(o1.bit(p))
        assert w[p >> 6] == 1 << (63 - (p & 63))
        assert sum(1 for x in w if x) == 1
    # lexicographic order = tuple order = integer order
    a, b = o1.bit(5), o1.bit(7)
    assert a > b and o1.words(a) > o1.words(b)


def test_fn3_printed_values():
    """PAPER.md:132 fn.3 prints ~1e-11 for (|S2|=10, d=3) and (5, 2)."""
    for line in golden_lines("fn3.txt"):
        m, k, s2, d, mag = map(int, line.split())
        v = o1.fp_fn3(m, k, s2, d)
        assert round(math.log10(v)) == mag, v
    # and the exact values the formula gives: 1.53e-11 and 1.27e-11
    assert o1.fp_fn3(192, 7, 10, 3) == pytest.approx(1.5334e-11, rel=1e-3)
    assert o1.fp_fn3(192, 7, 5, 2) == pytest.approx(1.2734e-11, rel=1e-3)


def test_fp_exact_brute_force_tiny():
    """fp_exact (the with-replacement expectation) equals full enumeration of
    all position tuples on tiny m, k."""
    for m, k, s2, d in [(6, 2, 1, 1), (5, 2, 2, 1), (4, 1, 2, 2), (7, 3, 1, 1)]:
        n2, n1 = k * s2, k * d
        hits = 0
        for b2 in itertools.product(range(m), repeat=n2):
            ones = set(b2)
            for b1 in itertools.product(range(m), repeat=n1):
                hits += all(x in ones for x in b1)
        assert o1.fp_exact(m, k, s2, d) == pytest.approx(hits / m ** (n2 + n1), rel=1e-12)


def test_fp_exact_approaches_fn3_for_wide_filters():
    """fn.3 is the large-m limit of the exact expectation."""
    for s2, d in [(10, 1), (20, 1), (5, 2)]:
        assert o1.fp_exact(19200, 7, s2 * 100, d) == pytest.approx(o1.fp_fn3(19200, 7, s2 * 100, d), rel=0.02)


@pytest.mark.parametrize("s2,d,trials", [(20, 1, 1_000_000), (15, 1, 1_000_000), (10, 1, 4_000_000)])
def test_encoder_false_positive_rate(s2, d, trials):
    """Monte Carlo FP rate of the encoder vs the exact fn.3-model expectation,
    +-5 sigma (a dropped probe, a wrong width or correlated probes fail it)."""
    fp, pop = o2.fp_montecarlo(seed=1000 + s2, s2=s2, d=d, trials=trials)
    p = o1.fp_exact(192, 7, s2, d)
    sigma = math.sqrt(p * (1 - p) / trials)
    assert abs(fp / trials - p) < 5 * sigma, (fp / trials, p, sigma)
    # mean popcount of sig(S2): m(1 - (1-1/m)^{k|S2|})
    e = o1.expected_popcount(192, 7, s2)
    assert abs(pop / trials - e) < 0.02 * e


def test_popcount_five_and_eight_tags():
    """5 tags -> 32.07 bits, 8 tags -> 48.68 bits on average."""
    for n, want in [(5, 32.07), (8, 48.68)]:
        assert o1.expected_popcount(192, 7, n) == pytest.approx(want, abs=0.01)
        fp, pop = o2.fp_montecarlo(seed=77 + n, s2=n, d=1, trials=200_000)
        assert pop / 200_000 == pytest.approx(want, abs=0.1)


def test_per_tag_popcount_at_most_k():
    rnd = random.Random(3)
    for _ in range(300):
        t = bytes(rnd.getrandbits(8) for _ in range(rnd.randrange(1, 20)))
        s = o1.encode([t])
        assert 1 <= bin(s).count("1") <= 7


# --------------------------------------------------------------- matching ---
def _tiny_universe(seed, n_vocab=40, n_sets=2000, n_q=500):
    rnd = random.Random(seed)
    vocab = [f"tag{i}".encode() for i in range(n_vocab)]
    sets = [frozenset(rnd.sample(range(n_vocab), rnd.randint(1, 5))) for _ in range(n_sets)]
    queries = [frozenset(rnd.sample(range(n_vocab), rnd.randint(6, 12))) for _ in range(n_q)]
    keys = [[rnd.randrange(300) for _ in range(rnd.randint(1, 3))] for _ in range(n_sets)]
    return vocab, sets, queries, keys


def test_zero_false_negatives_and_fp_excess():
    """S1 subset S2 => B1 subset B2 (no false negatives); the
    excess over exact containment is Bloom false positives, rare per fn.3."""
    vocab, sets, queries, keys = _tiny_universe(11)
    sigs = [o1.encode(vocab[t] for t in s) for s in sets]
    qs = [o1.encode(vocab[t] for t in q) for q in queries]
    got = set()
    for j, q in enumerate(qs):
        for i, s in enumerate(sigs):
            if o1.subset(s, q):
                got.add((j, i))
    exact = {(j, i) for j, q in enumerate(queries) for i, s in enumerate(sets) if s <= q}
    assert exact <= got
    excess = len(got - exact)
    # expected FPs: sum over non-contained pairs of P(FP) <= tiny; allow a few
    assert excess <= max(5, 0.01 * len(exact)), (excess, len(exact))
    # O1 match() output equals the (j, key) expansion of these pairs
    want = sorted((j, k) for j, i in got for k in keys[i])
    assert o1.match(sigs, keys, qs, unique=False) == want


def test_special_cases():
    """SURVEY 8c special cases: s = q matches; the empty set matches every
    query; the empty query matches only the empty set; an all-ones query
    matches everything; match-unique = unique(match)."""
    a = o1.encode([b"x", b"y"])
    b = o1.encode([b"x"])
    sigs = [a, b, 0, o1.FULL]
    keys = [[1], [2, 2], [3], [4]]
    assert o1.match(sigs, keys, [a], False) == [(0, 1), (0, 2), (0, 2), (0, 3)]
    assert o1.match(sigs, keys, [a], True) == [(0, 1), (0, 2), (0, 3)]
    assert o1.match(sigs, keys, [0], False) == [(0, 3)]
    assert o1.match(sigs, keys, [o1.FULL], False) == [(0, 1), (0, 2), (0, 2), (0, 3), (0, 4)]
    m = o1.match(sigs, keys, [a, b, 0], False)
    u = o1.match(sigs, keys, [a, b, 0], True)
    assert u == sorted(set(m))


def test_numpy_and_o2_match_equal_o1():
    vocab, sets, queries, keys = _tiny_universe(5, n_vocab=60, n_sets=700, n_q=150)
    sigs = [o1.encode(vocab[t] for t in s) for s in sets]
    qs = [o1.encode(vocab[t] for t in q) for q in queries]
    db_w = np.array([o1.words(s) for s in sigs], dtype=np.uint64)
    q_w = np.array([o1.words(q) for q in qs], dtype=np.uint64)
    key_off = np.zeros(len(keys) + 1, np.uint64)
    key_off[1:] = np.cumsum([len(k) for k in keys])
    flat = np.array([k for kl in keys for k in kl], np.uint32)
    for unique in (False, True):
        want = o1.match(sigs, keys, qs, unique)
        nq, nk = o1.match_numpy(db_w, key_off, flat, q_w, unique)
        assert list(zip(nq.tolist(), nk.tolist())) == want
        bq, bk = o2.match_brute(db_w, key_off, flat, q_w, unique, nthreads=3)
        assert list(zip(bq.tolist(), bk.tolist())) == want
        for max_p in (0xFFFFFFFF, 200, 50, 7, 1):
            ix = o2.Index(db_w, max_p)
            pq, pk, _ = ix.match(key_off, flat, q_w, unique, nthreads=2)
            assert list(zip(pq.tolist(), pk.tolist())) == want
        assert o1.match_partitioned(sigs, keys, qs, 25, unique) == want


# ---------------------------------------------------------- Algorithms 1,2,4 ---
def _parse_alg1_example():
    sets, parts, out = {}, [], {}
    for line in golden_lines("alg1_example.txt"):
        tok = line.split()
        if tok[0] == "max_p":
            out["max_p"] = int(tok[1])
        elif tok[0] == "set":
            sets[int(tok[1])] = [int(x) for x in tok[2:]]
        elif tok[0] == "part":
            lhs, rhs = line[4:].split("|")
            parts.append(([int(x) for x in lhs.split()], [int(x) for x in rhs.split()]))
        else:
            out[tok[0]] = [int(x) for x in tok[1:]]
    sigs = [sum(o1.bit(p) for p in sets[i]) for i in range(len(sets))]
    return sigs, parts, out


def test_alg1_hand_worked_example():
    sigs, parts, out = _parse_alg1_example()
    got = o1.alg1(sigs, out["max_p"])
    assert [(o1.positions(m), P) for m, P in got] == parts
    # O2 implements the same FIFO queue
    db_w = np.array([o1.words(s) for s in sigs], dtype=np.uint64)
    ix = o2.Index(db_w, out["max_p"])
    o2parts = []
    for i in range(ix.n_parts):
        m = o1.from_words(*ix.masks[i].tolist())
        mem = ix.members[ix.part_off[i]:ix.part_off[i + 1]].tolist()
        o2parts.append((o1.positions(m), mem))
    assert o2parts == parts


def test_alg2_hand_worked_example():
    sigs, parts, out = _parse_alg1_example()
    masks = [sum(o1.bit(p) for p in m) for m, _ in parts]
    PT = o1.partition_table(masks)
    q = sum(o1.bit(p) for p in out["query"])
    assert o1.alg2(PT, q) == out["routed"]
    matched = sorted(i for pi in o1.alg2(PT, q) for i in parts[pi][1] if o1.subset(sigs[i], q))
    assert matched == out["matches"]
    assert matched == [i for i, s in enumerate(sigs) if o1.subset(s, q)]


@pytest.mark.parametrize("max_p", [1, 3, 50, 400])
def test_alg1_invariants(max_p):
    """Every set in exactly one partition; mask subset of each member;
    |P| <= MAX_P unless all members are identical; mask never empty unless the
    partition is the zero partition (reading R7)."""
    vocab, sets, _, _ = _tiny_universe(21, n_vocab=50, n_sets=1500, n_q=1)
    sigs = [o1.encode(vocab[t] for t in s) for s in sets] + [0, 0]  # two empty sets
    parts = o1.alg1(sigs, max_p)
    seen = sorted(i for _, P in parts for i in P)
    assert seen == list(range(len(sigs)))
    for m, P in parts:
        assert all(o1.subset(m, sigs[i]) for i in P)
        if len(P) > max_p:
            assert len({sigs[i] for i in P}) == 1
        if m == 0:
            assert all(sigs[i] == 0 for i in P)
    # the O2 implementation computes the same table
    db_w = np.array([o1.words(s) for s in sigs], dtype=np.uint64)
    ix = o2.Index(db_w, max_p)
    assert ix.n_parts == len(parts)
    for i, (m, P) in enumerate(parts):
        assert o1.from_words(*ix.masks[i].tolist()) == m
        assert ix.members[ix.part_off[i]:ix.part_off[i + 1]].tolist() == P


def test_alg2_equals_brute_force_routing():
    """forward q to exactly the partitions with mask_i subset q."""
    vocab, sets, queries, _ = _tiny_universe(33, n_vocab=50, n_sets=1000, n_q=200)
    sigs = [o1.encode(vocab[t] for t in s) for s in sets] + [0]
    parts = o1.alg1(sigs, 20)
    masks = [m for m, _ in parts]
    PT = o1.partition_table(masks)
    for q in queries:
        qs = o1.encode(vocab[t] for t in q)
        assert sorted(o1.alg2(PT, qs)) == [i for i, m in enumerate(masks) if o1.subset(m, qs)]


def test_tile_prefix_hand_example_and_soundness():
    """Alg. 4: the common prefix of a lexicographically
    sorted run is contained in every set of the run."""
    first = sum(o1.bit(p) for p in (0, 3, 5))
    last = sum(o1.bit(p) for p in (0, 3, 7))
    assert o1.positions(o1.tile_prefix(first, last)) == [0, 3]
    assert o1.tile_prefix(first, first) == first
    rnd = random.Random(9)
    for _ in range(50):
        run = sorted(rnd.getrandbits(192) & rnd.getrandbits(192) & rnd.getrandbits(192) for _ in range(32))
        run.sort(reverse=True)   # any monotone run works; lexicographic = integer order
        for lo in range(0, 32, 8):
            tile = run[lo:lo + 8]
            tile.sort()
            pre = o1.tile_prefix(tile[0], tile[-1])
            assert all(o1.subset(pre, s) for s in tile)


def test_match_exact_definition():
    """O1.match_exact is plain set containment; on the tiny universe it is the
    Bloom result minus the false positives (soundness)."""
    vocab, sets, queries, keys = _tiny_universe(41, n_vocab=30, n_sets=800, n_q=120)
    ds = [[vocab[t] for t in s] for s in sets]
    qs = [[vocab[t] for t in q] for q in queries]
    ex = o1.match_exact(ds, keys, qs, False)
    bl = o1.match([o1.encode(s) for s in ds], keys, [o1.encode(q) for q in qs], False)
    want = sorted((j, k) for j, q in enumerate(queries) for i, s in enumerate(sets) if s <= q for k in keys[i])
    assert ex == want
    assert set(ex) <= set(bl)
