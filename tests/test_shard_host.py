"""Host-side logic of the multi-GPU path (CPU only): the library's host
Algorithm 1, the partition -> shard plan, owner ranges, and the exchange
protocol run by 2 processes over torch.distributed (gloo), with the oracle
standing in for the per-shard GPU match."""
import os
import socket

import numpy as np
import pytest

import tmgen
from oracle import o1, o2
from paper_conf_eurosys_rogorapkmcc17_b200 import _build, tagmatch as tm


@pytest.fixture(scope="module", autouse=True)
def lib():
    _build.build()
    tm.load()


@pytest.mark.parametrize("max_p", [1, 50, 500, 200_000, 0xFFFFFFFF])
def test_library_alg1_equals_oracle_alg1(c1, max_p):
    """tm_partition_host (the library's Alg. 1, no GPU) == O2's Alg. 1: same
    FIFO acceptance order, masks, sizes and member signatures."""
    sig = o2.encode(c1.db)
    masks, sizes, psig = tm.partition_host(sig, max_p)
    ix = o2.Index(sig, max_p)
    assert np.array_equal(masks, ix.masks)
    assert np.array_equal(sizes, np.diff(ix.part_off))
    off = 0
    for p in range(ix.n_parts):
        mem = sig[ix.members[ix.part_off[p]:ix.part_off[p + 1]].astype(np.int64)]
        mem = mem[np.lexsort((mem[:, 2], mem[:, 1], mem[:, 0]))]
        got = psig[off:off + int(sizes[p])]
        assert np.array_equal(got, mem)   # lexicographic inside the partition
        off += int(sizes[p])


def test_alg1_dedupes_identical_signatures():
    sig = np.array([[1, 0, 0], [1, 0, 0], [2, 0, 0], [0, 0, 0], [0, 0, 0]], np.uint64)
    masks, sizes, psig = tm.partition_host(sig, 1)
    assert int(sizes.sum()) == 3 and psig.shape[0] == 3


@pytest.mark.parametrize("G", [1, 2, 3, 8])
@pytest.mark.parametrize("routed", [False, True])
def test_shard_plan_contiguous_balanced_ranges(c1, G, routed):
    """tm_shard_plan: contiguous ranges of the partition table, deterministic, each
    shard's work within one partition's work of the fair share W/G (the midpoint rule)."""
    sig = o2.encode(c1.db)
    masks, sizes, _ = tm.partition_host(sig, 300)
    r = None
    if routed:   # weights from a routed query sample: Alg. 2 by brute force (the oracle's)
        qs = o2.encode(c1.queries)
        r = np.array([int(np.sum(np.all((m[None, :] & ~qs) == 0, axis=1))) for m in masks], np.uint64)
        w = sizes.astype(float) * r
    else:
        w = sizes * 0.25 ** np.array([sum(bin(int(x)).count("1") for x in m) for m in masks])
    own = tm.shard_plan(masks, sizes, G, r)
    assert own.shape[0] == masks.shape[0] and own.max() < G
    assert np.all(np.diff(own.astype(np.int64)) >= 0)                 # contiguous ranges, in order
    assert np.array_equal(own, tm.shard_plan(masks, sizes, G, r))    # deterministic
    load = np.array([w[own == g].sum() for g in range(G)])
    assert np.all(np.abs(load - w.sum() / G) <= w.max() + 1e-9)


def test_exchange_plan_offsets():
    """tm_exchange_plan: send offsets = prefix of the rank's row, receive offsets = prefix of its column."""
    rng = np.random.default_rng(5)
    for G in (1, 2, 3, 8):
        c = rng.integers(0, 1000, (G, G)).astype(np.uint64)
        for r in range(G):
            so, ro = tm.exchange_plan(c, r)
            assert np.array_equal(so, np.concatenate([[0], np.cumsum(c[r, :])]))
            assert np.array_equal(ro, np.concatenate([[0], np.cumsum(c[:, r])]))


@pytest.mark.parametrize("Q,G", [(0, 3), (1, 4), (100, 3), (100_000, 8), (7, 7)])
def test_owner_ranges_cover_queries(Q, G):
    r = [tm.owner_range(Q, G, g) for g in range(G)]
    assert r[0][0] == 0 and r[-1][1] == Q
    assert all(r[g][1] == r[g + 1][0] for g in range(G - 1))


# ---------------------------------------------------------------- gloo ---
def _shard_worker(rank, world, port, result):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        wl = tmgen.generate(3000, 400, seed=77)
        sig = o2.encode(wl.db)
        qsig = o2.encode(wl.queries)
        Q = qsig.shape[0]
        # every rank computes the same table and plan (no communication needed)
        masks, sizes, psig = tm.partition_host(sig, 100)
        own = tm.shard_plan(masks, sizes, world)
        plans = [torch.zeros(own.size, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(plans, torch.from_numpy(own.astype(np.int64)))
        same_plan = all(torch.equal(plans[0], p) for p in plans)
        # this shard's signatures -> its DB entries
        mine = set()
        off = 0
        for p, sz in enumerate(sizes.astype(int)):
            if own[p] == rank:
                mine.update(map(tuple, psig[off:off + sz].tolist()))
            off += sz
        ent = np.array([tuple(s) in mine for s in sig.tolist()])
        idx = np.nonzero(ent)[0]
        ko = np.zeros(idx.size + 1, np.uint64)
        ko[1:] = np.cumsum(wl.key_off[idx + 1] - wl.key_off[idx])
        ks = np.concatenate([wl.keys[wl.key_off[i]:wl.key_off[i + 1]] for i in idx]) if idx.size else \
            np.zeros(0, np.uint32)
        out = {}
        for unique in (False, True):
            # local match of this shard (the oracle stands in for the GPU scan)
            lq, lk = o2.match_brute(sig[idx], ko, ks, qsig, unique)
            pairs = (lq.astype(np.uint64) << np.uint64(32)) | lk.astype(np.uint64)
            # cut at the owner boundaries, all-gather the count matrix, then the library's
            # exchange plan (tm_exchange_plan) gives the send / receive offsets
            cuts = [tm.owner_range(Q, world, g) for g in range(world)]
            cnt = torch.tensor([int(np.sum((lq >= lo) & (lq < hi))) for lo, hi in cuts], dtype=torch.int64)
            allc = [torch.zeros(world, dtype=torch.int64) for _ in range(world)]
            dist.all_gather(allc, cnt)
            counts = np.stack([a.numpy() for a in allc]).astype(np.uint64)
            soff, roff = tm.exchange_plan(counts, rank)
            # grouped point-to-point send/recv, as ncclSend/ncclRecv in the library: the sorted
            # local pairs are the send buffer (owners are contiguous query ranges)
            rbuf = torch.zeros(int(roff[-1]), dtype=torch.int64)
            sbuf = torch.from_numpy(pairs.view(np.int64).copy())
            reqs = []
            for g in range(world):
                s0, s1 = int(soff[g]), int(soff[g + 1])
                r0, r1 = int(roff[g]), int(roff[g + 1])
                if g == rank:
                    rbuf[r0:r1] = sbuf[s0:s1]
                    continue
                if s1 > s0:
                    reqs.append(dist.isend(sbuf[s0:s1].clone(), g))
                if r1 > r0:
                    tmp = torch.zeros(r1 - r0, dtype=torch.int64)
                    reqs.append((dist.irecv(tmp, g), tmp, r0, r1))
            for rq in reqs:
                if isinstance(rq, tuple):
                    rq[0].wait()
                    rbuf[rq[2]:rq[3]] = rq[1]
                else:
                    rq.wait()
            recv = [rbuf]
            got = np.concatenate([r.numpy().view(np.uint64) for r in recv])
            got = np.sort(got)
            if unique:
                got = np.unique(got)
            # owner slice of the global oracle result
            wq, wk = o2.match_brute(sig, wl.key_off, wl.keys, qsig, unique)
            lo, hi = cuts[rank]
            sel = (wq >= lo) & (wq < hi)
            want = (wq[sel].astype(np.uint64) << np.uint64(32)) | wk[sel].astype(np.uint64)
            out[unique] = bool(np.array_equal(got, want)) and want.size > 0
        result[rank] = (same_plan, out[False], out[True])
    finally:
        dist.destroy_process_group()


def test_exchange_protocol_two_ranks_gloo():
    """World size 2 over gloo: plan agreement, owner cut, count all-gather,
    all-to-all of (q<<32|key) pairs and the owner-side merge reproduce the
    global result slice by slice, for match and match-unique."""
    import torch.multiprocessing as mp
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    mgr = mp.Manager()
    result = mgr.dict()
    mp.spawn(_shard_worker, args=(2, port, result), nprocs=2, join=True)
    assert dict(result) == {0: (True, True, True), 1: (True, True, True)}


def test_auto_max_partition_rule(c1):
    """TM_AUTO_MAX_PARTITION (R8b) resolves to clamp(n / 30,000, 5,000, 200,000): on the
    host hook the table equals the one built with that MAX_P given explicitly."""
    sig = o2.encode(c1.db)
    auto = tm.partition_host(sig, tm.TM_AUTO_MAX_PARTITION)
    want = min(200_000, max(5_000, sig.shape[0] // 30_000))
    explicit = tm.partition_host(sig, want)
    for a, b in zip(auto, explicit):
        assert np.array_equal(a, b)
