"""Partitioning (consolidate) time vs database size -- the Fig. 8 analogue (PAPER.md:375-381:
"about 50 seconds for the full workload of 200 million tag sets", MAX_P = 200K, CPU).
Here consolidate() runs on the GPU (tm_build.cu): the library's build_ms (H2D of the input,
encode, sort, distinct signatures, Alg. 1, row order, table / masks / keys) for N tag sets of
the Twitter-like workload, at MAX_P 200K (the paper's Fig. 8) and auto; plus, at smaller N, the
mutable path (tm_add_sets staging + tm_consolidate).

usage: python scripts/build_time.py [N list, e.g. 10000000,30000000,100000000,300000000]
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import tmgen  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def main():
    ns = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "10000000,30000000,100000000,300000000").split(",")]
    for n in ns:
        t = time.time()
        wl = tmgen.generate(n, 1000, seed=3)
        gen_s = time.time() - t
        for mp in (200_000, tmb.TM_AUTO_MAX_PARTITION):
            t = time.time()
            db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp, tile_filter=1, row_order=1)
            wall = time.time() - t
            st = db.stats()
            db.close()
            print(json.dumps({"n_sets": n, "max_partition": st["max_partition"], "build_ms": st["build_ms"],
                              "wall_s": wall, "partitions": st["n_partitions"], "rows": st["n_rows"],
                              "gen_s": gen_s, "path": "tm_build"}), flush=True)
        if n <= 5_000_000:
            db = tmb.Database.create(max_partition=200_000, tile_filter=1, row_order=1)
            t = time.time()
            db.add_sets(wl.db, wl.key_off, wl.keys)
            stage_s = time.time() - t
            t = time.time()
            db.consolidate()
            cons_s = time.time() - t
            st = db.stats()
            db.close()
            print(json.dumps({"n_sets": n, "max_partition": 200_000, "stage_s": stage_s, "consolidate_s": cons_s,
                              "build_ms": st["build_ms"], "partitions": st["n_partitions"],
                              "path": "tm_add_sets + tm_consolidate"}), flush=True)
        del wl


if __name__ == "__main__":
    main()
