"""One warm match call of a config under `ncu --profile-from-start off`: the kernels of exactly one
call (cudaProfilerStart/Stop around it), for per-kernel stage times.
usage: ncu --profile-from-start off --metrics gpu__time_duration.sum --csv python scripts/stage_probe.py C3 5000"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import tmgen  # noqa: E402
import paper_conf_eurosys_rogorapkmcc17_b200 as tmb  # noqa: E402


def main():
    cfg, mp = sys.argv[1], int(sys.argv[2])
    os.environ.setdefault("TM_SCAN_VARIANT", "14")
    wl = tmgen.config(cfg)
    q = wl.queries
    arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64),
                                              q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
    dt = [torch.from_numpy(a).cuda() for a in arrs]
    dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                            arrs[0].size, arrs[1].size - 1, arrs[2].size, q.n_sets)
    stream = torch.cuda.current_stream()
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=mp, tile_filter=1, row_order=1)
    for _ in range(2):
        db.match_batch_device(dq, False, stream.cuda_stream)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    db.match_batch_device(dq, False, stream.cuda_stream)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(db.stats())
    db.close()


if __name__ == "__main__":
    main()
