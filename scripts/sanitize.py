"""Run every scan-kernel variant (TM_SCAN_VARIANT) on small workloads for compute-sanitizer
(memcheck / racecheck / synccheck): C1 (10K sets x 1K queries, one partition and MAX_P 500) and
a 100K-set slice at MAX_P 5000, match and match-unique, plus the streaming (<= 8 queries) and
sharded-merge paths.  Each result is compared with the oracle's brute force, so a run that the
sanitizer does not flag is also a parity run.

usage: compute-sanitizer --tool <tool> python scripts/sanitize.py [variants] [n_sets]
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import tmgen  # noqa: E402
from oracle import o2  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def check(db, q, db_sig, wl, unique, what):
    gq, gk = db.match_batch(q, unique)
    wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, o2.encode(q), unique)
    ok = np.array_equal(gq, wq) and np.array_equal(gk, wk)
    print(f"{what}: {gq.size} pairs {'ok' if ok else 'MISMATCH'}", flush=True)
    if not ok:
        raise SystemExit(1)


def main():
    variants = (sys.argv[1] if len(sys.argv) > 1 else "0,5,6,7,8,9,10,11,12,13,14,15,16").split(",")
    big = int(sys.argv[2]) if len(sys.argv) > 2 else 100_000
    cases = [("C1", tmgen.config("C1"), [(tmb.TM_NO_PARTITIONING, 2), (500, 1), (500, 0)]),
             (f"{big}", tmgen.generate(big, 2000, seed=11, max_partition=5000), [(5000, 1)])]
    for name, wl, layouts in cases:
        db_sig = o2.encode(wl.db)
        for mp, filt in layouts:
            with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp, tile_filter=filt,
                              row_order=1 if filt == 1 else 0) as db:
                for v in variants:
                    os.environ["TM_SCAN_VARIANT"] = v
                    for unique in (False, True):
                        check(db, wl.queries, db_sig, wl, unique, f"{name} maxp={mp} filter={filt} var={v} u={unique}")
                    small = wl.queries.subset(np.arange(5))
                    check(db, small, db_sig, wl, False, f"{name} maxp={mp} filter={filt} var={v} Q=5")
    os.environ.pop("TM_SCAN_VARIANT", None)
    # in-process multi-GPU handles (peer-copy exchange, owner merge) and a mutable handle
    wl = tmgen.generate(big, 2000, seed=12, max_partition=5000)
    db_sig = o2.encode(wl.db)
    for mode in (0, 1):
        with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=5000, tile_filter=1, row_order=1, n_gpus=2,
                          device_ids=[0, 0], shard_mode=mode) as db:
            for unique in (False, True):
                check(db, wl.queries, db_sig, wl, unique, f"group mode={mode} u={unique}")
    db = tmb.Database.create(max_partition=5000, tile_filter=1, row_order=1)
    db.add_sets(wl.db, wl.key_off, wl.keys)
    db.consolidate()
    check(db, wl.queries, db_sig, wl, False, "mutable: add_sets + consolidate")
    db.close()
    print("sanitize run complete")


if __name__ == "__main__":
    main()
