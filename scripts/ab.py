"""In-process A/B of scan-kernel variants (TM_SCAN_VARIANT) and MAX_P values on one workload,
the same inputs and the same box, with a bit-exact check of every configuration against the
first one (and optionally the oracle on a sample).

usage: python scripts/ab.py <config> "<variants, e.g. 5,8>" ["<max_partition list, e.g. 200000,20000>"] [reps]
prints one JSON line per (max_partition, variant): median scan / route / total ms, stats.
"""
import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import tmgen  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def main():
    cfg = sys.argv[1]
    variants = [v for v in sys.argv[2].split(",") if v]
    maxps = [int(x) for x in (sys.argv[3].split(",") if len(sys.argv) > 3 and sys.argv[3] else ["0"])]
    reps = int(sys.argv[4]) if len(sys.argv) > 4 else 5
    filt = int(os.environ.get("AB_FILTER", "1"))
    order = int(os.environ.get("AB_ROW_ORDER", "1" if filt == 1 else "0"))
    t0 = time.time()
    wl = tmgen.config(cfg)
    gen_s = time.time() - t0
    q = wl.queries
    arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64),
                                              q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
    dt = [torch.from_numpy(a).cuda() for a in arrs]
    dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                            arrs[0].size, arrs[1].size - 1, arrs[2].size, q.n_sets)
    stream = torch.cuda.current_stream()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    ref = None
    for mp in maxps:
        t0 = time.time()
        db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp or wl.max_partition, tile_filter=filt,
                          row_order=order)
        build_s = time.time() - t0
        for v in variants:
            if v == "auto":
                os.environ.pop("TM_SCAN_VARIANT", None)
            else:
                os.environ["TM_SCAN_VARIANT"] = v
            for _ in range(16):
                db.match_batch_device(dq, False, stream.cuda_stream)
                if not db.stats()["tuning"]:
                    break
            for _ in range(2):
                db.match_batch_device(dq, False, stream.cuda_stream)
            sts = []
            for _ in range(reps):
                flush.zero_()
                db.match_batch_device(dq, False, stream.cuda_stream)
                sts.append(db.stats())
            gq, gk = db.match_batch(q, False)
            key = (gq.astype(np.uint64) << np.uint64(32)) | gk.astype(np.uint64)
            h = int(np.bitwise_xor.reduce(key * np.uint64(0x9E3779B97F4A7C15))) if key.size else 0
            if ref is None:
                ref = (key.size, h)
            same = (key.size, h) == ref
            med = {k: statistics.median(s[k] for s in sts) for k in ("scan_ms", "route_ms", "encode_ms",
                                                                      "merge_ms", "total_ms")}
            st = sts[-1]
            print(json.dumps({"config": cfg, "max_partition": mp or wl.max_partition, "variant": v,
                              "ran_variant": st["scan_variant"], **med,
                              "q_per_s": q.n_sets / (med["total_ms"] / 1e3),
                              "n_partitions": st["n_partitions"], "routed": st["routed"],
                              "candidate_pairs": st["candidate_pairs"], "tile_tests": st["tile_tests"],
                              "pair_checks": st["pair_checks"], "work_items": st["work_items"],
                              "pairs": int(key.size), "same_as_first": same, "build_s": build_s,
                              "gen_s": gen_s}), flush=True)
        db.close()
    os.environ.pop("TM_SCAN_VARIANT", None)


if __name__ == "__main__":
    main()
