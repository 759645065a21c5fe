"""Offline filter-hierarchy experiment (CPU, test infrastructure only): how many
(set, query) pair checks survive AND masks of 32-row tiles vs 8/16-row groups
in the balanced-split row order (R18), on a sample of C2 partitions.

Usage: python scripts/sim_filters.py [n_sets] [n_queries] [n_parts_sampled]
"""
import sys

import numpy as np

sys.path.insert(0, __file__.rsplit("/scripts/", 1)[0])
import tmgen  # noqa: E402
from oracle import o2  # noqa: E402
from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tmb  # noqa: E402


def bits(s):
    """[n,3] u64 -> [n,192] bool, position p = word p>>6, bit 63-(p&63)."""
    b = s.astype(">u8").view(np.uint8).reshape(-1, 24)
    return np.unpackbits(b, axis=1).astype(bool)


def refine(sb, idx, leaf=8):
    out = []
    st = [idx]
    while st:
        r = st.pop()
        if r.size <= leaf:
            out.append(r)
            continue
        f = sb[r].sum(0)
        cand = (f > 0) & (f < r.size)
        if not cand.any():
            out.append(r)
            continue
        d = np.abs(2 * f.astype(np.int64) - r.size)
        d[~cand] = 1 << 40
        pv = int(np.argmin(d))
        on = sb[r, pv]
        st.append(r[on])
        st.append(r[~on])
    return np.concatenate(out)


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
    nq = int(sys.argv[2]) if len(sys.argv) > 2 else 20_000
    nps = int(sys.argv[3]) if len(sys.argv) > 3 else 6
    wl = tmgen.generate(n, nq, seed=2)
    sig = np.unique(o2.encode(wl.db), axis=0)
    qs = o2.encode(wl.queries)
    masks, sizes, usig = tmb.partition_host(sig, 200_000)
    print(f"{usig.shape[0]} distinct sigs, {masks.shape[0]} partitions")
    off = np.concatenate([[0], np.cumsum(sizes.astype(np.int64))])
    qb = bits(qs)
    rng = np.random.default_rng(0)
    tot = {}
    w = sizes.astype(np.float64) / sizes.sum()
    for p in rng.choice(masks.shape[0], size=min(nps, masks.shape[0]), replace=False, p=w):
        ps = usig[off[p]:off[p + 1]]
        sb = bits(ps)
        order = refine(sb, np.arange(ps.shape[0]))
        sb = sb[order]
        mb = bits(masks[p:p + 1])[0]
        routed = ~(qb[:, mb] == False).any(1)  # mask within q
        qr = qb[routed]
        nz = ~qr  # query zero bits
        res = {"sets": sb.shape[0], "routed": int(routed.sum())}
        for g in (256, 32, 16, 8, 4, 1):
            ng = (sb.shape[0] + g - 1) // g
            pad = ng * g - sb.shape[0]
            sbp = np.concatenate([sb, np.ones((pad, 192), bool)]) if pad else sb
            andm = sbp.reshape(ng, g, 192).all(1)
            # pass[q, group] = andm within q  <=> no bit of andm in the zero bits of q
            fail = (nz.astype(np.uint8) @ andm.T.astype(np.uint8)) > 0
            npass = int((~fail).sum())
            res[g] = (npass, npass * g, float(andm.sum(1).mean()))
            if g == 8:
                # quarter-warp layout: per (32-row tile, 128-query unit), the longest of the tile's
                # four group lists bounds the loop; B = tile-32 survivors (for comparison)
                passg = ~fail  # [q, group]
                nt = (ng + 3) // 4
                pg = np.zeros((passg.shape[0], nt * 4), bool)
                pg[:, :ng] = passg
                pg = pg.reshape(passg.shape[0], nt, 4)
                mx = 0
                tb = 0
                for u in range(0, pg.shape[0], 128):
                    blk = pg[u:u + 128]
                    mx += int(blk.sum(0).max(1).sum())
                res["qw_max"] = (mx, mx * 32, 0.0)
        for k, v in res.items():
            if isinstance(v, tuple):
                tot.setdefault(k, [0, 0])
                tot[k][0] += v[0]
                tot[k][1] += v[1]
        print(p, res)
    print("totals (group passes, pair checks implied):")
    for k, v in tot.items():
        print(f"  group {k!s:>6}: passes {v[0]:.3e} pair checks {v[1]:.3e}")


if __name__ == "__main__":
    main()
