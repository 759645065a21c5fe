"""Per-call scan-kernel times and variants of repeated device-API calls on one handle (tuning
round, then steady state), with and without an L2 flush before each call.
usage: python scripts/scan_timeline.py [config] [calls]"""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import tmgen  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C3"
    calls = int(sys.argv[2]) if len(sys.argv) > 2 else 12
    t0 = time.time()
    wl = tmgen.config(name)
    print(f"{name}: generated in {time.time() - t0:.1f} s", flush=True)
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=wl.max_partition, device=0, tile_filter=1,
                      row_order=1)
    q = wl.queries
    arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64), q.tag_idx.view(np.int32),
                                              q.set_off.view(np.int64))]
    dt = [torch.from_numpy(a).cuda() for a in arrs]
    dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                            arrs[0].size, arrs[1].size - 1, arrs[2].size, q.n_sets)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    nvml = os.environ.get("TL_NVML", "")   # "clock", "reasons", "both": poll NVML every 20 ms from call 6 on
    import threading
    stop = threading.Event()

    def poll():
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(0)
        while not stop.is_set():
            if nvml in ("clock", "both"):
                pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
            if nvml in ("reasons", "both"):
                pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
            time.sleep(0.02)
    th = None
    e2e = os.environ.get("TL_E2E", "") == "1"   # interleave host-API calls (as bench.py's warm-up does)
    hq = tmb.HostTagSets(q.vocab_bytes, q.vocab_off, q.tag_idx, q.set_off) if e2e else None
    for i in range(calls):
        if e2e and i < 6:
            pr = db.match_batch_raw(hq, False)
            db.free_pairs(pr)
            st = db.stats()
            print(f"e2e  {i:2d} variant {st['scan_variant']} scan {st['scan_ms']:8.2f} ms", flush=True)
        if nvml and i == 6:
            th = threading.Thread(target=poll, daemon=True)
            th.start()
        fl = i % 2 == 1
        if fl:
            flush.zero_()
        t = time.perf_counter()
        db.match_batch_device(dq, False, s.cuda_stream)
        torch.cuda.synchronize()
        st = db.stats()
        print(f"call {i:2d} flush={int(fl)} variant {st['scan_variant']} scan {st['scan_ms']:8.2f} ms total "
              f"{st['total_ms']:8.2f} ms wall {(time.perf_counter() - t) * 1e3:8.2f} ms items {st['work_items']}",
              flush=True)
    stop.set()
    db.close()


if __name__ == "__main__":
    main()
