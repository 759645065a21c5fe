"""Subset-scan HBM roofline sweep (BASELINE metric "subset-scan HBM
GB/s vs roofline"): the whole table as ONE partition (MAX_P = no partitioning),
the pre-filter off, and batches of B queries; every stored signature is read
from HBM once per call (24 B/set) and checked against the B queries.  Small B
is HBM-bound, large B ALU-bound.

usage: python scripts/hbm_sweep.py [n_sets] [filters]   -> JSON lines on stdout
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
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402
from oracle import o2  # noqa: E402


def main():
    n_sets = int(sys.argv[1]) if len(sys.argv) > 1 else 100_000_000
    filters = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "2").split(",")]
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    hbm = float(peaks["hbm_gbs"])
    t0 = time.time()
    wl = tmgen.generate(n_sets, 4096, seed=3)
    gen_s = time.time() - t0
    stream = torch.cuda.current_stream()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    db_sig = None
    for filt in filters:
        t0 = time.time()
        db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=tmb.TM_NO_PARTITIONING, tile_filter=filt)
        build_s = time.time() - t0
        rows = db.stats()["n_rows"]
        for B, var in [(int(b), v) for b in os.environ.get("HBM_B", "1,2,4,8,16,32,64,128,256").split(",")
                       for v in os.environ.get("HBM_VARIANTS", "auto").split(",")]:
            if var == "auto":
                os.environ.pop("TM_SCAN_VARIANT", None)
            else:
                os.environ["TM_SCAN_VARIANT"] = var
            q = wl.queries.subset(np.arange(B))
            arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64),
                                                      q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
            dt = [torch.from_numpy(a).cuda() for a in arrs]
            dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                                    arrs[0].size, arrs[1].size - 1, arrs[2].size, B)
            for _ in range(16):   # warm-up, then until the handle has tuned this batch size
                db.match_batch_device(dq, False, stream.cuda_stream)
                if not db.stats()["tuning"]:
                    break
            for _ in range(2):
                db.match_batch_device(dq, False, stream.cuda_stream)
            scan = []
            for _ in range(5):
                flush.zero_()          # the table (2.4 GB at 100M) exceeds L2 anyway
                db.match_batch_device(dq, False, stream.cuda_stream)
                scan.append(db.stats()["scan_ms"])
            st = db.stats()
            ms = float(np.median(scan))
            table_bytes = 24 * rows
            gbs = table_bytes / (ms / 1e3) / 1e9
            if db_sig is None:
                db_sig = o2.encode(wl.db)
            ok = None
            if True:   # brute-force parity of the B queries at every B (<= 256 queries: seconds)
                gq, gk = db.match_batch(q, False)
                wq, wk = o2.match_brute(db_sig, wl.key_off, wl.keys, o2.encode(q), False)
                ok = bool(np.array_equal(gq, wq) and np.array_equal(gk, wk))
            print(json.dumps({"B": B, "forced": var, "tile_filter": filt, "n_sets": n_sets, "rows": rows, "scan_ms": ms,
                              "table_gbs": gbs, "frac_of_measured_hbm": gbs / hbm,
                              "pair_checks": st["pair_checks"], "tile_tests": st["tile_tests"],
                              "checks_per_s": st["pair_checks"] / (ms / 1e3), "parity": ok,
                              "variant": st["scan_variant"], "work_items": st["work_items"],
                              "gen_s": gen_s, "build_s": build_s}), flush=True)
        db.close()


if __name__ == "__main__":
    main()
