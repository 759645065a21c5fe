"""Latency vs batch timeout (Fig. 6 analogue; NEXT-2): an
open-loop Poisson stream of queries is replayed into a tm_stream at a fixed
rate; batches close at max_batch queries or when the oldest query has waited
the timeout.  Reports throughput and the latency distribution (submit -> result
published) per timeout.

usage: python scripts/stream_latency.py <config> <rate q/s> <n queries> <timeouts_us,...> [max_batch]
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
from paper_conf_eurosys_rogorapkmcc17_b200.tagmatch import Stream  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
    rate = float(sys.argv[2]) if len(sys.argv) > 2 else 1e6
    nq = int(sys.argv[3]) if len(sys.argv) > 3 else 200_000
    timeouts = [int(x) for x in (sys.argv[4] if len(sys.argv) > 4 else "500,1000,2000,5000").split(",")]
    max_batch = int(sys.argv[5]) if len(sys.argv) > 5 else 1 << 20
    c = dict(tmgen.CONFIGS[cfg])
    mp = int(os.environ.get("STREAM_MAX_PARTITION", str(tmb.TM_AUTO_MAX_PARTITION)))  # bench.py's default
    wl = tmgen.generate(c["n_sets"], max(nq, c["n_queries"]), c["seed"])
    q = wl.queries.subset(np.arange(nq))
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp, tile_filter=1, row_order=1)
    db.match_batch(q, True)          # warm-up: grow every device / pinned buffer once
    for b in (1, 8, 100, 1000, 3000, 10000):   # and load the kernels small batches use (CUB
        db.match_batch(q.subset(np.arange(min(b, nq))), True)  # single-tile sorts; lazy loading)
    rng = np.random.default_rng(7)
    arrivals = np.cumsum(rng.exponential(1e9 / rate, nq)).astype(np.uint64)
    for to in timeouts:
        with Stream(db, max_batch, to, unique=True) as st:
            t0 = time.time()
            st.replay(q, arrivals)
            st.flush()
            lat, sizes, first_sub, last_done = [], [], None, 0
            service, wait_disp = [], []
            while (r := st.poll(wait=False)) is not None:
                lat.append(r["done_ns"] - r["submit_ns"])
                sizes.append(r["tickets"].size)
                service.append((r["done_ns"] - r["dispatch_ns"]) / 1e6)          # the GPU call
                wait_disp.append((r["dispatch_ns"] - r["submit_ns"].min()) / 1e6)  # oldest query's wait
                first_sub = r["submit_ns"].min() if first_sub is None else min(first_sub, r["submit_ns"].min())
                last_done = max(last_done, r["done_ns"])
            lat = np.concatenate(lat) / 1e6
            sizes = np.array(sizes)
            print(json.dumps({"config": cfg, "rate_qps": rate, "n_queries": nq, "timeout_us": to,
                              "max_batch": max_batch, "throughput_qps": nq / ((last_done - first_sub) / 1e9),
                              "latency_ms_p50": float(np.percentile(lat, 50)),
                              "latency_ms_p99": float(np.percentile(lat, 99)), "latency_ms_max": float(lat.max()),
                              "batches": int(sizes.size), "mean_batch": float(sizes.mean()),
                              "service_ms_max": float(max(service)), "service_ms_p50": float(np.median(service)),
                              "dispatch_wait_ms_max": float(max(wait_disp)),
                              "slowest_batch": int(sizes[int(np.argmax(service))]),
                              "wall_s": time.time() - t0}), flush=True)
    db.close()


if __name__ == "__main__":
    main()
