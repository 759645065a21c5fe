"""C5: query tag-count sweep at 100M tag sets (BASELINE config 4; PAPER.md:288-306,
Fig. 2/3 analogue): input throughput (queries/s) and output throughput (pairs/s)
vs query size, on one B200, with a sampled bit-exact parity check per point.

usage: python scripts/sweep_c5.py [n_sets] [n_queries] [steps]  -> JSON lines on stdout
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import tmgen  # noqa: E402
from oracle import o2  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def main():
    n_sets = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000_000
    n_q = int(sys.argv[2]) if len(sys.argv) > 2 else 100_000
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    totals = list(range(2, 21, 2))
    t0 = time.time()
    wl, batches, _ = tmgen.generate_sweep(n_sets, 500, n_q, totals, 500)
    gen_s = time.time() - t0
    t0 = time.time()
    # the layout bench.py times: balanced splits inside partitions + tile AND masks (DESIGN R17/R18)
    mp = int(os.environ.get("C5_MAX_PARTITION", str(tmb.TM_AUTO_MAX_PARTITION)))  # bench.py's default
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp, tile_filter=1, row_order=1)
    build_s = time.time() - t0
    db_sig = o2.encode(wl.db)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()
    for t in totals:
        q = batches[t]
        arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64),
                                                  q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
        dt = [torch.from_numpy(a).cuda() for a in arrs]
        dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                                arrs[0].size, arrs[1].size - 1, arrs[2].size, q.n_sets)
        for unique in (True, False):
            for _ in range(16):   # warm-up, then until the handle has tuned this batch size
                db.match_batch_device(dq, unique, stream.cuda_stream)
                if not db.stats()["tuning"]:
                    break
            for _ in range(2):
                db.match_batch_device(dq, unique, stream.cuda_stream)
            ms = []
            for _ in range(steps):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                out = db.match_batch_device(dq, unique, stream.cuda_stream)
                b.record(stream)
                torch.cuda.synchronize()
                ms.append(a.elapsed_time(b))
            st = db.stats()
            # sampled parity (64 queries, brute force over the whole database)
            gq, gk = db.match_batch(q, unique)
            rng = np.random.default_rng(t)
            qsel = np.sort(rng.choice(q.n_sets, 64, replace=False))
            wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, o2.encode(q.subset(qsel)), unique,
                                    qid=qsel.astype(np.uint32))
            keep = np.isin(gq, qsel)
            ok = bool(np.array_equal(gq[keep], wq) and np.array_equal(gk[keep], wk))
            mean_ms = float(np.mean(ms))
            print(json.dumps({"tags_per_query": t, "mode": "match-unique" if unique else "match",
                              "queries_per_s": q.n_sets / (mean_ms / 1e3), "ms_per_batch": mean_ms,
                              "pairs_per_query": out.n / q.n_sets, "output_pairs_per_s": out.n / (mean_ms / 1e3),
                              "scan_ms": st["scan_ms"], "candidate_pairs": st["candidate_pairs"],
                              "pair_checks": st["pair_checks"], "routed_per_query": st["routed"] / q.n_sets,
                              "sample_parity": ok, "n_sets": n_sets, "n_queries": q.n_sets,
                              "scan_variant": st["scan_variant"], "layout": "tile-and + balanced-splits",
                              "max_partition": db.stats()["max_partition"],
                              "gen_s": gen_s, "build_s": build_s}), flush=True)
    db.close()


if __name__ == "__main__":
    main()
