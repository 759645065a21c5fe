"""Offline experiment (CPU, test infrastructure only): row-order rules inside partitions and
the strength of 32-row tile AND masks (the level-B filter) -- pair checks implied by the tile
masks for a query sample, per rule.  Rules for the recursive split inside a partition (DESIGN.md
R18 uses "balanced": the unused bit whose frequency is closest to 50%):
  balanced   freq closest to 1/2
  frac=F     freq closest to F (F > 1/2 favours a large side sharing the pivot bit)
usage: python scripts/sim_order.py [n_sets] [n_queries] [max_p] [rules, e.g. balanced,frac=0.7]
"""
import sys

import numpy as np

sys.path.insert(0, __file__.rsplit("/scripts/", 1)[0])
import tmgen  # noqa: E402
from oracle import o2  # noqa: E402
from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tmb  # noqa: E402


def bits(s):
    b = s.astype(">u8").view(np.uint8).reshape(-1, 24)
    return np.unpackbits(b, axis=1).astype(bool)


def refine(sb, idx, target, leaf=8):
    out, st = [], [idx]
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
        d = np.abs(f.astype(np.float64) - target * r.size)
        d[~cand] = 1e18
        pv = int(np.argmin(d))
        on = sb[r, pv]
        st.append(r[on])
        st.append(r[~on])
    return np.concatenate(out)


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
    nq = int(sys.argv[2]) if len(sys.argv) > 2 else 4000
    maxp = int(sys.argv[3]) if len(sys.argv) > 3 else 5000
    rules = (sys.argv[4] if len(sys.argv) > 4 else "balanced,frac=0.6,frac=0.7,frac=0.8").split(",")
    wl = tmgen.generate(n, nq, seed=2)
    sig = np.unique(o2.encode(wl.db), axis=0)
    qs = o2.encode(wl.queries)
    masks, sizes, usig = tmb.partition_host(sig, maxp)
    off = np.concatenate([[0], np.cumsum(sizes.astype(np.int64))])
    qb = bits(qs)
    nz = (~qb).astype(np.float32)
    tot = {r: [0, 0] for r in rules}
    for p in range(masks.shape[0]):
        ps = usig[off[p]:off[p + 1]]
        mb = bits(masks[p:p + 1])[0]
        routed = ~(qb[:, mb] == False).any(1)
        if not routed.any():
            continue
        nzr = nz[routed]
        sb0 = bits(ps)
        for r in rules:
            t = 0.5 if r == "balanced" else float(r.split("=")[1])
            sb = sb0[refine(sb0, np.arange(ps.shape[0]), t)]
            ng = (sb.shape[0] + 31) // 32
            pad = ng * 32 - sb.shape[0]
            sbp = np.concatenate([sb, np.ones((pad, 192), bool)]) if pad else sb
            andm = sbp.reshape(ng, 32, 192).all(1).astype(np.float32)
            passes = int(((nzr @ andm.T) == 0).sum())
            tot[r][0] += passes
            tot[r][1] += passes * 32
    print(f"n={n} queries={nq} max_p={maxp} partitions={masks.shape[0]}")
    for r, (a, b) in tot.items():
        print(f"  {r:12s} tile passes {a:.4e}  pair checks {b:.4e}  (x{b / tot[rules[0]][1]:.3f})")


if __name__ == "__main__":
    main()
