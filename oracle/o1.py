"""ORACLE O1 -- the plain definition of TagMatch's result, in Python.

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this module.  The product path
(the CUDA library) never imports it and shares no code with it.

Every function cites the passage it follows (PAPER.md line numbers, section /
algorithm / footnote).  Readings of silent or garbled passages are DESIGN.md
readings R1..R16.

Signature representation: a Python int S of 192 bits where position p
(0 <= p < 192) is bit (191 - p).  Word w of the C layout is
(S >> (128 - 64*w)) & (2**64 - 1), so position p lives in word p >> 6 at bit
63 - (p & 63) (reading R3), "leftmost" = lowest position, and lexicographic
order of signatures = integer order of S.

Parity status:
  * encoder: the hash choice is a reading (R1) -- "parity unpinned" against the
    paper, which names no hash.  Its primitives are pinned to published test
    vectors (FNV-1a-64, SplitMix64) and its statistics to fn.3.
  * match / match_unique: pinned by exact-containment brute force, special cases.
  * alg1 / alg2 / tile_prefix: pinned by invariants and a hand-worked example
    (tests/golden/alg1_example.txt).
"""
from __future__ import annotations

import math
from collections import deque
from typing import Iterable, Sequence

M = 192          # Bloom filter width
K = 7            # number of hash functions
MASK64 = (1 << 64) - 1
FULL = (1 << M) - 1

FNV_OFFSET = 0xCBF29CE484222325   # FNV-1a 64-bit offset basis (reading R1)
FNV_PRIME = 0x100000001B3         # FNV 64-bit prime
GOLDEN = 0x9E3779B97F4A7C15       # SplitMix64 increment


# ------------------------------------------------------------------ encoder --
def fnv1a64(data: bytes) -> int:
    """FNV-1a, 64 bit: h ^= byte; h *= prime (reading R1)."""
    h = FNV_OFFSET
    for b in data:
        h ^= b
        h = (h * FNV_PRIME) & MASK64
    return h


def splitmix64(state: int) -> tuple[int, int]:
    """One SplitMix64 step: returns (new_state, output)."""
    state = (state + GOLDEN) & MASK64
    z = state
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return state, z ^ (z >> 31)


def tag_positions(tag: bytes) -> list[int]:
    """The k = 7 bit positions of one tag (hash per reading R1/R2):
    the first 7 SplitMix64 outputs seeded with FNV-1a-64(tag), each mapped to
    [0, 192) by floor(z * 192 / 2^64).  Drawn with replacement (fn.3 model)."""
    state = fnv1a64(tag)
    out = []
    for _ in range(K):
        state, z = splitmix64(state)
        out.append((z * M) >> 64)
    return out


def bit(p: int) -> int:
    """Signature with only position p set."""
    return 1 << (M - 1 - p)


def encode(tags: Iterable[bytes]) -> int:
    """sig(T): OR over the tags of T of their 7 positions."""
    s = 0
    for t in tags:
        for p in tag_positions(t):
            s |= bit(p)
    return s


def words(s: int) -> tuple[int, int, int]:
    """The three 64-bit blocks of a signature (3 x 64-bit blocks)."""
    return ((s >> 128) & MASK64, (s >> 64) & MASK64, s & MASK64)


def from_words(w0: int, w1: int, w2: int) -> int:
    return (int(w0) << 128) | (int(w1) << 64) | int(w2)


def positions(s: int) -> list[int]:
    return [p for p in range(M) if s & bit(p)]


def subset(a: int, b: int) -> bool:
    """Bitwise inclusion a subset-of b, i.e. (a & ~b) == 0 (fn.4 read per R4)."""
    return (a & ~b & FULL) == 0


# ------------------------------------------------------------------ matching --
def match(db_sigs: Sequence[int], key_lists: Sequence[Sequence[int]], q_sigs: Sequence[int],
          unique: bool) -> list[tuple[int, int]]:
    """The definition: for query j, every key k of every entry
    (s, k) with sig(s) subset-of sig(q_j).  match: multiset, match-unique: set.
    Output sorted by (j, k) (reading R12)."""
    out = []
    for j, q in enumerate(q_sigs):
        ks = []
        for s, kl in zip(db_sigs, key_lists):
            if subset(s, q):
                ks.extend(kl)
        ks.sort()
        if unique:
            ks = sorted(set(ks))
        out.extend((j, k) for k in ks)
    return out


def match_numpy(db_w, key_off, keys, q_w, unique: bool, qids=None):
    """Same definition, vectorised over the database with numpy (one query at a
    time; the subset test (s & ~q) == 0 per 64-bit block).
    db_w: uint64 [N,3]; q_w: uint64 [Q,3].  Returns (q uint32[], key uint32[])."""
    import numpy as np
    db_w = np.asarray(db_w, dtype=np.uint64)
    q_w = np.asarray(q_w, dtype=np.uint64)
    key_off = np.asarray(key_off, dtype=np.int64)
    keys = np.asarray(keys, dtype=np.uint32)
    oq, ok = [], []
    for j in range(q_w.shape[0]):
        q = q_w[j]
        hit = ((db_w[:, 0] & ~q[0]) | (db_w[:, 1] & ~q[1]) | (db_w[:, 2] & ~q[2])) == 0
        idx = np.nonzero(hit)[0]
        if idx.size:
            ks = np.concatenate([keys[key_off[i]:key_off[i + 1]] for i in idx])
        else:
            ks = np.zeros(0, np.uint32)
        ks = np.unique(ks) if unique else np.sort(ks)
        oq.append(np.full(ks.size, j if qids is None else qids[j], np.uint32))
        ok.append(ks.astype(np.uint32))
    if not oq:
        return np.zeros(0, np.uint32), np.zeros(0, np.uint32)
    return np.concatenate(oq), np.concatenate(ok)


def match_exact(db_sets: Sequence[Iterable[bytes]], key_lists: Sequence[Sequence[int]],
                queries: Sequence[Iterable[bytes]], unique: bool) -> list[tuple[int, int]]:
    """Exact subset matching on the tag strings themselves (s_i
    subset of q; "an additional exact subset check"): for query j, every
    key of every entry whose tag set is contained in the query's tag set.
    Brute force over Python sets."""
    sets = [frozenset(s) for s in db_sets]
    out = []
    for j, q in enumerate(queries):
        qs = frozenset(q)
        ks = []
        for s, kl in zip(sets, key_lists):
            if s <= qs:
                ks.extend(kl)
        ks = sorted(set(ks)) if unique else sorted(ks)
        out.extend((j, k) for k in ks)
    return out


# ------------------------------------------------- Algorithm 1 --
def alg1(sigs: Sequence[int], max_p: int) -> list[tuple[int, list[int]]]:
    """Balanced partitioning, Algorithm 1, as written, with
    reading R7 for the cases the paper leaves open and R8 for "no partitioning".

    Returns the partition table as a list of (mask, member indices) in the
    order partitions are accepted from the FIFO work queue Q."""
    if max_p == 0xFFFFFFFF:
        return [(0, list(range(len(sigs))))] if sigs else []
    PT = []
    Q = deque([(0, list(range(len(sigs))), 0)])   # (mask -> P, used_bits)
    while Q:
        mask, P, used = Q.popleft()
        if not P:                                   # R7: empty P dropped
            continue
        if len(P) <= max_p and mask != 0:
            PT.append((mask, P))
            continue
        freq = [0] * M                              # frequencies of one-bits in P
        for i in P:
            for p in positions(sigs[i]):
                freq[p] += 1
        cands = [p for p in range(M) if not (used & bit(p)) and 0 < freq[p] < len(P)]
        if not cands:                               # R7: all members equal sigma
            PT.append((sigs[P[0]], P))
            continue
        # pivot: unused bit with frequency closest to 50%; ties -> lowest position (R7)
        pivot = min(cands, key=lambda p: (abs(2 * freq[p] - len(P)), p))
        P0 = [i for i in P if not (sigs[i] & bit(pivot))]
        P1 = [i for i in P if sigs[i] & bit(pivot)]
        used |= bit(pivot)
        Q.append((mask, P0, used))
        Q.append((mask | bit(pivot), P1, used))
    return PT


# ------------------------------------------------- Algorithm 2 --
def leftmost(s: int) -> int | None:
    """Position of the leftmost one-bit (lowest position), None if s == 0."""
    if s == 0:
        return None
    return M - s.bit_length()


def partition_table(masks: Sequence[int]) -> list[list[tuple[int, int]]]:
    """PT[j] = [(mask_i, i)] for masks whose leftmost one-bit is j;
    PT[192] holds empty masks, forwarded to every query (reading R9)."""
    PT = [[] for _ in range(M + 1)]
    for i, m in enumerate(masks):
        j = leftmost(m)
        PT[M if j is None else j].append((m, i))
    return PT


def alg2(PT, q: int) -> list[int]:
    """Pre-process stage, Algorithm 2: for each one-bit j of
    q, for each (mask_i -> P_i) in PT[j]: if mask_i subset-of q, forward q to P_i."""
    out = []
    for j in positions(q) + [M]:
        for m, i in PT[j]:
            if subset(m, q):
                out.append(i)
    return out


def match_partitioned(db_sigs, key_lists, q_sigs, max_p: int, unique: bool):
    """The paper's pipeline on one core: Alg. 1, Alg. 2, then a linear scan of
    every routed partition (Alg. 3 semantics), key lookup
     and merge.  Equal to match() by construction."""
    parts = alg1(db_sigs, max_p)
    PT = partition_table([m for m, _ in parts])
    out = []
    for j, q in enumerate(q_sigs):
        ks = []
        for pi in alg2(PT, q):
            for i in parts[pi][1]:
                if subset(db_sigs[i], q):
                    ks.extend(key_lists[i])
        ks = sorted(set(ks)) if unique else sorted(ks)
        out.extend((j, k) for k in ks)
    return out


# ------------------------------------------------- Algorithm 4 --
def tile_prefix(first: int, last: int) -> int:
    """Alg. 4 with reading R6: len = leftmost nonzero bit of
    first XOR last; prefix = first with all positions >= len cleared.  If
    first == last the prefix is the whole signature."""
    x = first ^ last
    if x == 0:
        return first
    ln = leftmost(x)
    return first & ~((1 << (M - ln)) - 1)


# ------------------------------------------------- fn. 3 false positives ------
def fp_fn3(m: int, k: int, s2: int, d: int) -> float:
    """P(B1 subset B2) = (1 - e^{-k|S2|/m})^{k|S1\\S2|} (footnote 3)."""
    return (1.0 - math.exp(-k * s2 / m)) ** (k * d)


def fp_exact(m: int, k: int, s2: int, d: int) -> float:
    """Exact with-replacement false-positive probability under the same model
    as fn.3 (k*|S2| independent uniform positions fill B2; each of the k*d
    positions of S1\\S2 must land on a one-bit of B2): E[(X/m)^{k d}] with X the
    number of distinct positions hit by k*|S2| draws (occupancy distribution)."""
    n = k * s2
    dist = [0.0] * (m + 1)
    dist[0] = 1.0
    for _ in range(n):
        nd = [0.0] * (m + 1)
        for x, p in enumerate(dist):
            if p == 0.0:
                continue
            nd[x] += p * x / m
            if x < m:
                nd[x + 1] += p * (m - x) / m
        dist = nd
    return sum(p * (x / m) ** (k * d) for x, p in enumerate(dist))


def expected_popcount(m: int, k: int, n_tags: int) -> float:
    """E[popcount(sig(T))] for |T| = n_tags distinct tags: m (1 - (1 - 1/m)^{k n})."""
    return m * (1.0 - (1.0 - 1.0 / m) ** (k * n_tags))
