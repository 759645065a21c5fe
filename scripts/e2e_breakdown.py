"""Where the end-to-end (host buffers in, host pairs out) time of a C2 call goes: wall time of
tm_match_batch vs tm_match_batch_device on resident queries, and the bare H2D / D2H copies of the
same bytes.  usage: python scripts/e2e_breakdown.py [n_sets] [n_queries]"""
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import tmgen  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def wall(fn, n=10):
    ts = []
    for _ in range(n):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        ts.append((time.perf_counter() - t0) * 1e3)
    return statistics.median(ts)


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
    Q = int(sys.argv[2]) if len(sys.argv) > 2 else 100_000
    wl = tmgen.generate(n, Q, seed=2)
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=200_000, device=0, tile_filter=1, row_order=1)
    qarr = [np.ascontiguousarray(a) for a in (wl.queries.vocab_bytes, wl.queries.vocab_off.view(np.int64),
                                              wl.queries.tag_idx.view(np.int32), wl.queries.set_off.view(np.int64))]
    dt = [torch.from_numpy(a).cuda() for a in qarr]
    pinned = [torch.from_numpy(a).pin_memory() for a in qarr]
    dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                            qarr[0].size, qarr[1].size - 1, qarr[2].size, Q)
    hq = tmb.HostTagSets(pinned[0].numpy(), pinned[1].numpy().view(np.uint64), pinned[2].numpy().view(np.uint32),
                         pinned[3].numpy().view(np.uint64))
    s = torch.cuda.current_stream()

    def dev():
        db.match_batch_device(dq, False, s.cuda_stream)

    def e2e():
        p = db.match_batch_raw(hq, False)
        db.free_pairs(p)

    for _ in range(8):
        dev()
        e2e()
    st = db.stats()
    npairs = st["result_pairs"]
    out_d = torch.empty(2 * npairs, dtype=torch.int32, device="cuda")
    out_h = torch.empty(2 * npairs, dtype=torch.int32, pin_memory=True)

    def h2d():
        for d, h in zip(dt, pinned):
            d.copy_(h, non_blocking=True)

    def d2h():
        out_h.copy_(out_d, non_blocking=True)

    r = {"device_call_ms": wall(dev), "e2e_call_ms": wall(e2e), "h2d_ms": wall(h2d), "d2h_ms": wall(d2h),
         "h2d_bytes": sum(a.nbytes for a in qarr), "d2h_bytes": 8 * npairs}
    st = db.stats()
    r.update({k: st[k] for k in ("encode_ms", "route_ms", "scan_ms", "merge_ms", "total_ms")})
    print(r)


if __name__ == "__main__":
    main()
