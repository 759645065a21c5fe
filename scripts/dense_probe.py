"""One-partition dense-scan probe for ncu: the C3-size table (100M sets) as ONE partition with the
pre-filter off, B queries, forced scan variant; three calls (ncu: capture the last).
usage: python scripts/dense_probe.py B variant"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import tmgen  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402

B, var = int(sys.argv[1]), sys.argv[2]
os.environ["TM_SCAN_VARIANT"] = var
wl = tmgen.generate(100_000_000, 4096, seed=3)
with tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=tmb.TM_NO_PARTITIONING, tile_filter=2) as db:
    q = wl.queries.subset(np.arange(B))
    for _ in range(3):
        db.match_batch(q, False)
    st = db.stats()
    print(B, var, st["scan_variant"], st["scan_ms"], st["pair_checks"])
