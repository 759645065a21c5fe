#!/usr/bin/env python
"""bench.py -- TagMatch B200 throughput (driver contract).

A step = one tm_match_batch over one batch of queries = the whole hot path
(encode, route, batch, pre-filter, subset scan, compaction,
key expansion, sort/merge).  Default workload: N = 1 -> BASELINE config C3
(100M tag sets, 1M-query stream, MAX_P = 200K: the largest single-GPU config);
N > 1 -> C4 (300M tag sets) partition-sharded over the N ranks; `match`
(Table 1).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C3] [--unique]

value  : queries/s over all ranks, inputs resident in HBM (tm_match_batch_device),
         per-step CUDA events on the launching stream, L2 flushed between steps.
e2e    : queries/s through tm_match_batch_csr with pinned host queries (H2D inside
         the timed region) and the result -- every query's sorted keys -- copied
         back to host (D2H: 4 B per pair + 8 B per query offset).
hbm    : (N = 1) the subset scan of the whole table as ONE partition, pre-filter off,
         B = 1 / 4 / 16 queries: table bytes / scan-kernel time vs the measured HBM
         copy bandwidth (the BASELINE metric's "subset-scan HBM GB/s vs roofline").
roofline: the dominant kernel (k_scan) against the INT/logic-pipe peak measured on
         this box by build/int_peak (scripts/int_peak.cu), SURVEY 8(d) ops model.
N > 1  : one process per GPU (torchrun), the same batch on every rank, "scaling": "strong".
         Default: the database is partition-sharded over the ranks (plan
         weighted by a routed 10K-query sample): every rank matches the batch against its
         partitions and the pairs go to query owners over NCCL (tm_match_batch_sharded_device).
         --replicated: every rank holds the whole database and matches its owner range of the
         batch, no exchange (NEXT-1; the library's TM_SHARD_REPLICATED).
MAX_P  : auto (TM_AUTO_MAX_PARTITION: clamp(N / 3*10^4, 5K, 200K), R8b) unless
         --max-partition N (--max-partition 200000 = the paper's value).
--impl reference : the oracle (oracle/o2.c, the paper's CPU method) on the
         host cores, on a bounded sample of the same workload per step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "queries/sec vs DB size at 1/2/4/8 B200; subset-scan HBM GB/s vs roofline"
ALU_LANES_PER_SM_CLK = 64     # fallback only: LOP3 ALU pipe 16 lanes/clk/SMSP x 4 (B300_MICROARCH.md)
SM_COUNT = 148
# SURVEY.md 8(d) per-unit figures (the primary roofline model): a pre-filter test (mask vs
# query, Alg. 4) = 4 INT ops, a pair check (set vs query, Alg. 3: 6 LOP3 + 1 ISETP) = 7
SURVEY_OPS_PER_TILE_TEST = 4
SURVEY_OPS_PER_PAIR_CHECK = 7
# secondary model: the minimum one 64-bit block test per decision = 3 ops
MIN_OPS_PER_DECISION = 3


class _CAI:
    """__cuda_array_interface__ view of a library-owned device array (uint32)."""

    def __init__(self, ptr, n, typestr="<u4"):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """Samples SM clock and throttle reasons with NVML during the timed region."""

    def __init__(self, device_index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            pass
        self._stop = threading.Event()
        self._t = None

    _REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
                0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks_setting",
                0x1: "gpu_idle", 0x100: "display_clock_setting", 0x10: "sync_boost"}

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self._REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def load_workload(name: str, rank: int = 0):
    """BASELINE config `name`; rank r > 0 matches its own query batch (query seed + 7919 r)."""
    import tmgen
    if name in tmgen.CRAFTED:  # sec. 4.4 crafted workloads
        mp = getattr(load_workload, "max_partition", -1)
        c = dict(tmgen.CRAFTED[name], max_partition=0xFFFFFFFE if mp == -1 else (mp or 200_000), total_tags=0,
                 oracle_max_partition=200_000)
        c["resolved_max_partition"] = min(200_000, max(5_000, c["n_sets"] // 30_000))
        wl = tmgen.config(name, max_partition=c["max_partition"],
                          query_seed=c["seed"] + (1 << 32) + 7919 * rank)
        return wl, c
    c = dict(tmgen.CONFIGS[name])
    c["oracle_max_partition"] = c["max_partition"]   # O2's own MAX_P (the paper's 200K)
    mp = getattr(load_workload, "max_partition", -1)
    if mp == -1:
        c["max_partition"] = 0xFFFFFFFE   # TM_AUTO_MAX_PARTITION
        c["resolved_max_partition"] = min(200_000, max(5_000, c["n_sets"] // 30_000))  # the library's rule
    elif mp:
        c["max_partition"] = mp
    wl = tmgen.generate(c["n_sets"], c["n_queries"], c["seed"], total_tags=c["total_tags"],
                        max_partition=c["max_partition"], name=name,
                        query_seed=(c.get("query_seed") or c["seed"] + (1 << 32)) + 7919 * rank)
    return wl, c


# ------------------------------------------------------------------ oracle --
def oracle_rate(wl, c, unique: bool, target_s: float = 8.0, max_q: int | None = None):
    """O2 (the paper's CPU method: Alg. 1 + Alg. 2 + linear scan, std threads)
    on a bounded query sample sized for ~target_s seconds."""
    from oracle import o2
    db_sig = o2.encode(wl.db)
    q_sig = o2.encode(wl.queries)
    t0 = time.perf_counter()
    if c["n_sets"] <= 20_000_000:
        ix = o2.Index(db_sig, c.get("oracle_max_partition", 200_000))
    else:
        # O2's single-threaded Alg. 1 takes minutes beyond ~20M sets (213 s at 100M):
        # the baseline is then O2's brute-force scan on all cores
        ix = _BruteOracle(db_sig)
    build_s = time.perf_counter() - t0
    nq = q_sig.shape[0]
    n = min(nq, 256 if isinstance(ix, o2.Index) else 32)
    t0 = time.perf_counter()
    ix.match(wl.key_off, wl.keys, q_sig[:n], unique)
    dt = max(time.perf_counter() - t0, 1e-6)
    per_q = dt / n
    size = int(min(nq, max(n, target_s / per_q)))
    if max_q:
        size = min(size, max_q)
    return ix, q_sig, size, build_s


class _BruteOracle:
    """O2 brute force with the Index.match signature."""
    kind = "brute force"

    def __init__(self, db_sig):
        self.db = db_sig

    def match(self, key_off, keys, q_sig, unique, qid=None):
        from oracle import o2
        q, k = o2.match_brute(self.db, key_off, keys, q_sig, unique, qid=qid)
        return q, k, (0, 0)


def run_reference(args):
    """--impl reference: the oracle as it stands, rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import o2
    wl, c = load_workload(args.config)
    unique = bool(args.unique)
    ix, q_sig, size, build_s = oracle_rate(wl, c, unique, target_s=args.ref_step_s)
    rng = np.random.default_rng(0)
    times = []
    for step in range(args.warmup + args.steps):
        sel = np.sort(rng.choice(q_sig.shape[0], size, replace=False))
        t0 = time.perf_counter()
        ix.match(wl.key_off, wl.keys, q_sig[sel], unique, qid=sel.astype(np.uint32))
        dt = time.perf_counter() - t0
        if step >= args.warmup:
            times.append(dt)
    tot = sum(times)
    value = size * len(times) / tot
    cores = o2.threads(0)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * tot / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
            "data": ("synthetic (seeded sec. 4.4 crafted workload, tmgen.generate_crafted, PAPER.md:391-399)"
                     if args.config.startswith(("C6", "C7")) else
                     "synthetic (seeded Twitter-like generator tmgen, PAPER.md:258-282)"),
            "config": config_block(c, args, wl, args.gpus > 1),
            "cpu_baseline": {"value": value, "unit": "queries/s", "cores": cores, "kind": "oracle",
                             "sample": f"{size} of {q_sig.shape[0]} queries per step ("
                                       + (f"O2 brute force over {c['n_sets']} sets" if isinstance(ix, _BruteOracle)
                                          else f"O2: Alg.1 MAX_P={c.get('oracle_max_partition')} + Alg.2 + linear scan; "
                                               f"Alg.1 build {build_s:.1f} s excluded") + ")"},
            "e2e": {"value": value, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_block(c, args, wl, sharded=False):
    return {"workload": args.config, "n_sets": c["n_sets"], "n_queries": c["n_queries"],
            "query_tags": (f"{c['set_tags']}-tag DB sets, {c['query_tags']}-tag queries (PAPER.md:391-399)"
                           if "set_tags" in c else
                           "base set + 2..4 extra" if not c["total_tags"] else f"total {c['total_tags']}"),
            "max_partition": (f"auto: clamp(N/3e4, 5000, 200000) = {c['resolved_max_partition']}"
                              if c["max_partition"] == 0xFFFFFFFE else c["max_partition"]),
            "mode": "match-unique" if args.unique else "match",
            "tile_filter": ["alg4-prefix", "tile-and", "none"][args.tile_filter],
            "row_order": ["lexicographic", "balanced-splits"][args.row_order],
            "exact_check": bool(args.exact),
            "parallelism": (f"replicated-{args.gpus} (each rank: owner range of the batch, whole table)"
                            if args.replicated else f"partition-sharded-{args.gpus} (NCCL exchange)")
                           if args.gpus > 1 else "single",
            "l2": "flushed between timed steps (512 MiB write)", "bloom": "192 bits, k=7 (PAPER.md:106)"}


def memory_block(db, mem0, mem1, dev):
    """Fig. 9 analogue: device memory the library holds, from
    cudaMemGetInfo deltas minus torch's own reservations (the library allocates with
    cudaMallocAsync, so pool memory it keeps counts): after tm_build (the database: tagset
    table, masks, key CSR) and after the timed calls (plus the per-call work buffers)."""
    import torch
    torch.cuda.synchronize(dev)
    free2, res2 = torch.cuda.mem_get_info(dev)[0], torch.cuda.memory_reserved(dev)
    st = db.stats()
    lib_db = (mem0[0] - mem1[0]) - (mem1[1] - mem0[1])
    lib_all = (mem0[0] - free2) - (res2 - mem0[1])
    return {"device_db_bytes": int(lib_db), "device_after_calls_bytes": int(lib_all),
            "tagset_table_bytes": int(st["n_rows"]) * 24, "key_table_bytes": int(st["n_entries"]) * 4,
            "note": "the key table lives on the GPU (the paper keeps it on the host, P:387)"}


# --------------------------------------------------------------------- ours --
def int_peak(peaks):
    """INT/logic-pipe peak of this GPU: scripts/int_peak.cu (built by build() as build/int_peak)
    run now on this GPU (LOP3 thread-ops per SM per clock, x SMs x the max SM clock); else the
    committed measurement profiles/int_peak.json; else the guide's 64 lanes/clk/SM."""
    import subprocess
    mhz = peaks.get("sm_max_mhz", 1965.0)
    res, src = None, None
    exe = os.path.join(ROOT, "build", "int_peak")
    if os.path.exists(exe):
        try:
            out = subprocess.run([exe], capture_output=True, text=True, timeout=60).stdout.strip().splitlines()
            res, src = json.loads(out[-1]), "measured now (build/int_peak)"
        except Exception:
            res = None
    if res is None:
        try:
            with open(os.path.join(ROOT, "profiles", "int_peak.json")) as f:
                res, src = json.load(f), "measured earlier (profiles/int_peak.json)"
        except Exception:
            res = None
    if res is None:
        return SM_COUNT * ALU_LANES_PER_SM_CLK * mhz * 1e6 / 1e12, \
            f"fallback: {SM_COUNT} SMs x {ALU_LANES_PER_SM_CLK} lanes/clk (B300_MICROARCH.md) x {mhz} MHz", None
    per_clk = res["lop3"]["ops_per_clk_per_sm"]
    return res["sms"] * per_clk * mhz * 1e6 / 1e12, \
        (f"{src}: LOP3 {per_clk:.1f} thread-ops/clk/SM x {res['sms']} SMs x {mhz} MHz (MEASURED_PEAKS.json "
         f"sm_max_mhz); measured {res['lop3']['tops']:.2f} Tops/s at ~{res['lop3']['sm_mhz_est']:.0f} MHz"), res


def ncu_traffic(config: str, variant: int, build_id: str):
    """DRAM traffic of k_scan from the committed ncu capture of this config, only if it was
    taken on the same library build (tm_build_id) and scan variant; else None + why."""
    path = os.path.join(ROOT, "profiles", f"ncu_scan_traffic_{config}.json")
    vpath = os.path.join(ROOT, "profiles", f"ncu_scan_traffic_{config}_v{variant}.json")
    if os.path.exists(vpath):   # a capture of this variant (the handle's tuner may settle on either)
        path = vpath
    try:
        with open(path) as f:
            tr = json.load(f)
    except Exception:
        return None, None, f"no committed ncu capture for {config}"
    if tr.get("build_id") != build_id or tr.get("variant") != variant:
        return None, None, (f"committed capture {os.path.basename(path)} is from build {tr.get('build_id')} "
                            f"variant {tr.get('variant')}, this run is build {build_id} variant {variant}")
    ncu = {k: tr.get(k) for k in ("alu_pipe_pct", "issue_active_pct", "warps_active_pct", "l2_hit_pct")}
    ncu["report"] = tr.get("report")
    return tr.get("dram_bytes_per_launch"), ncu, "same build and variant"


def hbm_block(wl, dev, stream, flush, Bs=(1, 4, 16)):
    """The subset scan of the whole table as ONE partition (no partitioning), pre-filter off:
    every stored signature read from HBM once per call (24 B/set) and checked against B queries
    (SURVEY 8(d) roofline sweep; the table is larger than L2)."""
    import torch
    import paper_conf_eurosys_rogorapkmcc17_b200 as tmb
    peaks, src = measured_peaks()
    hbm = float(peaks["hbm_gbs"])
    t0 = time.perf_counter()
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=tmb.TM_NO_PARTITIONING, device=dev,
                      tile_filter=2, row_order=0)
    build_s = time.perf_counter() - t0
    rows = db.stats()["n_rows"]
    pts = []
    for B in Bs:
        q = wl.queries.subset(np.arange(B))
        arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64),
                                                  q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
        dt = [torch.from_numpy(a).to(f"cuda:{dev}") for a in arrs]
        dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                                arrs[0].size, arrs[1].size - 1, arrs[2].size, B)
        for _ in range(16):
            db.match_batch_device(dq, False, stream.cuda_stream)
            if not db.stats()["tuning"]:
                break
        for _ in range(3):
            db.match_batch_device(dq, False, stream.cuda_stream)
        scan = []
        for _ in range(7):
            flush.zero_()
            db.match_batch_device(dq, False, stream.cuda_stream)
            scan.append(db.stats()["scan_ms"])
        st = db.stats()
        ms = statistics.median(scan)
        gbs = 24 * rows / (ms / 1e3) / 1e9
        pts.append({"B": B, "scan_ms": ms, "GB/s": gbs, "frac": gbs / hbm, "variant": st["scan_variant"],
                    "pair_checks_per_s": st["pair_checks"] / (ms / 1e3)})
    db.close()
    return {"table": f"whole {args_config_name(wl)} table as one partition, {rows} rows x 24 B = "
                     f"{24 * rows / 1e9:.2f} GB (> 126 MB L2), pre-filter off",
            "peak_gbs": hbm, "peak_src": f"{src} MEASURED_PEAKS.json hbm_gbs (read+write copy)",
            "timing": "median of 7 calls, CUDA events around the k_scan launch on the library stream, "
                      "L2 flushed before each", "points": pts, "build_s": build_s}


def args_config_name(wl):
    return getattr(wl, "name", "")


def run_ours(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # control-plane process group (barriers, max-over-ranks timing): NCCL, one GPU per
    # rank; TM_BENCH_PG=gloo allows a functional multi-rank run on a single GPU
    pg = os.environ.get("TM_BENCH_PG", "nccl")
    if world > 1:
        torch.cuda.set_device(local % torch.cuda.device_count())
        if pg == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local % torch.cuda.device_count()))
        else:
            dist.init_process_group(pg)
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()
    cdev = f"cuda:{dev}" if pg == "nccl" else "cpu"

    import __graft_entry__
    __graft_entry__.build() if rank == 0 or world == 1 else None
    if world > 1:
        dist.barrier()
    import paper_conf_eurosys_rogorapkmcc17_b200 as tmb
    from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tmx

    # N > 1: one batch on every rank; partitioned (default) or replicated database (library
    # shard_mode: each rank matches its owner range of the batch against the whole table)
    sharded = world > 1
    mode = tmx.TM_SHARD_REPLICATED if args.replicated else tmx.TM_SHARD_PARTITIONED
    wl, c = load_workload(args.config, 0)
    unique = bool(args.unique)
    Q = wl.queries.n_sets
    peaks, peak_src = measured_peaks()
    ipeak, ipeak_src, ipeak_raw = int_peak(peaks) if rank == 0 else (None, None, None)
    stream = torch.cuda.current_stream()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=f"cuda:{dev}")

    # the scaling base of a sharded run: the same workload on ONE GPU (rank 0), same steps
    base = None
    if sharded and rank == 0 and not args.no_scaling_base:
        base = single_gpu_value(wl, c, args, dev, stream, flush)
    if world > 1:
        dist.barrier()

    torch.cuda.synchronize(dev)
    mem0 = (torch.cuda.mem_get_info(dev)[0], torch.cuda.memory_reserved(dev))
    t0 = time.perf_counter()
    # the shard plan weighs partitions by the routing of a 10K-query sample of the stream
    sample = wl.queries.subset(np.arange(min(10_000, Q))) if sharded else None
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=c["max_partition"], device=dev,
                      tile_filter=args.tile_filter, row_order=args.row_order, exact=int(args.exact),
                      n_shards=world if sharded else 1, shard=rank if sharded else 0, shard_mode=mode,
                      plan_sample=sample)
    build_s = time.perf_counter() - t0
    c["resolved_max_partition"] = db.stats()["max_partition"]
    torch.cuda.synchronize(dev)
    mem1 = (torch.cuda.mem_get_info(dev)[0], torch.cuda.memory_reserved(dev))
    if sharded and mode == tmx.TM_SHARD_PARTITIONED:
        uid = [tmx.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        db.comm_init(uid[0], world, rank)

    # device-resident query batch (value) and pinned host copy (e2e)
    qarr = [np.ascontiguousarray(a) for a in (wl.queries.vocab_bytes, wl.queries.vocab_off.view(np.int64),
                                              wl.queries.tag_idx.view(np.int32), wl.queries.set_off.view(np.int64))]
    dt_ = [torch.from_numpy(a).to(f"cuda:{dev}") for a in qarr]
    dq = tmb.device_tagsets(dt_[0].data_ptr(), dt_[1].data_ptr(), dt_[2].data_ptr(), dt_[3].data_ptr(),
                            qarr[0].size, qarr[1].size - 1, qarr[2].size, Q)
    pinned = [torch.from_numpy(a).pin_memory() for a in qarr]
    hq = tmb.HostTagSets(pinned[0].numpy(), pinned[1].numpy().view(np.uint64), pinned[2].numpy().view(np.uint32),
                         pinned[3].numpy().view(np.uint64))
    h2d_bytes = sum(a.nbytes for a in qarr)

    def step_device():
        torch.cuda.nvtx.range_push("bench_device")   # ncu selects the device step's launches by this range
        try:
            if sharded:
                return db.match_batch_sharded_device(dq, unique, stream.cuda_stream)
            return db.match_batch_device(dq, unique, stream.cuda_stream)
        finally:
            torch.cuda.nvtx.range_pop()

    def step_e2e():
        """Public API end to end: host queries in, host pairs out; returns D2H bytes."""
        if not sharded:   # per-query key lists: 4 B per pair + 8 B per query come back
            p = db.match_batch_csr_raw(hq, unique)
            n = p.n
            db.free_csr(p)
            return n * 4 + (Q + 1) * 8
        for d, h in zip(dt_, pinned):          # H2D of the batch (every rank receives it)
            d.copy_(h, non_blocking=True)
        out = db.match_batch_sharded_device(dq, unique, stream.cuda_stream)
        if out.n:                              # D2H of this rank's owner slice
            host = torch.empty(2 * out.n, dtype=torch.int32, pin_memory=True)
            qt = torch.as_tensor(_CAI(out.query, out.n), device=f"cuda:{dev}")
            kt = torch.as_tensor(_CAI(out.key, out.n), device=f"cuda:{dev}")
            host[:out.n].copy_(qt)
            host[out.n:].copy_(kt)
        return out.n * 8

    tune_calls = finish_tuning(db, step_device, world, cdev)
    for _ in range(args.warmup):
        step_device()
        step_e2e()
    torch.cuda.synchronize()

    # ---- value: device-resident inputs, per-step CUDA events, L2 flushed between steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    launches, stats = 0, []
    sampler = ClockSampler(dev)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with sampler:
        for i in range(args.steps):
            flush.zero_()
            ev[i][0].record(stream)
            step_device()
            ev[i][1].record(stream)
            st = db.stats()
            launches += st["kernel_launches"]
            stats.append(st)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    t_local = sum(step_ms) / 1000.0
    t_max = t_local
    if world > 1:
        t = torch.tensor([t_local], device=cdev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t_max = float(t.item())
    value = Q * args.steps / t_max
    scan_ms = [s["scan_ms"] for s in stats]

    # per-rank view (sharded: scan time, exchange, imbalance)
    ranks = None
    if world > 1:
        mine = torch.tensor([statistics.mean(scan_ms), t_local * 1000 / args.steps,
                             statistics.mean(s["xchg_ms"] for s in stats),
                             statistics.mean(s["local_ms"] for s in stats),
                             float(stats[-1]["xchg_send_bytes"]), float(stats[-1]["xchg_recv_bytes"]),
                             float(stats[-1]["pair_checks"]), float(stats[-1]["n_rows"])],
                            device=cdev, dtype=torch.float64)
        allr = [torch.zeros_like(mine) for _ in range(world)]
        dist.all_gather(allr, mine)
        allr = [r.cpu().tolist() for r in allr]
        sc = [r[0] for r in allr]
        ranks = {"scan_ms": sc, "step_ms": [r[1] for r in allr], "xchg_ms": [r[2] for r in allr],
                 "local_ms": [r[3] for r in allr], "xchg_send_bytes": [int(r[4]) for r in allr],
                 "xchg_recv_bytes": [int(r[5]) for r in allr], "pair_checks": [int(r[6]) for r in allr],
                 "rows": [int(r[7]) for r in allr],
                 "scan_imbalance_max_over_mean": max(sc) / max(statistics.mean(sc), 1e-9)}

    # ---- e2e: host API, pinned inputs, H2D + D2H inside the timed region
    e2e_t, d2h = [], 0
    for i in range(args.steps):
        flush.zero_()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        d2h = step_e2e() + 8 * 2
        torch.cuda.synchronize()
        e2e_t.append(time.perf_counter() - t0)
    e2e_local = sum(e2e_t)
    if world > 1:
        t = torch.tensor([e2e_local], device=cdev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_local = float(t.item())
    e2e_value = Q * args.steps / e2e_local

    mem = memory_block(db, mem0, mem1, dev)
    db.close()
    hbm = None
    if world == 1 and not args.no_hbm:
        hbm = hbm_block(wl, dev, stream, flush)

    if rank == 0:
        last = stats[-1]
        scan_s = statistics.mean(scan_ms) / 1000.0
        ops = SURVEY_OPS_PER_TILE_TEST * last["tile_tests"] + SURVEY_OPS_PER_PAIR_CHECK * last["pair_checks"]
        ops_min = MIN_OPS_PER_DECISION * (last["tile_tests"] + last["pair_checks"])
        achieved = ops / scan_s / 1e12
        traffic, ncu, traffic_note = ncu_traffic(args.config, last["scan_variant"], tmx.build_id())
        line = {
            "metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": statistics.mean(step_ms), "higher_is_better": True,
            "scaling": "strong" if sharded else "weak", "vs_baseline": None, "dtype": "u64",
            "data": ("synthetic (seeded sec. 4.4 crafted workload, tmgen.generate_crafted, PAPER.md:391-399)"
                     if args.config.startswith(("C6", "C7")) else
                     "synthetic (seeded Twitter-like generator tmgen, PAPER.md:258-282)"),
            "config": config_block(c, args, wl, sharded),
            "roofline": {"bound": "alu", "achieved": achieved, "peak": ipeak, "unit": "Tops/s",
                         "frac": achieved / ipeak, "traffic": traffic, "traffic_note": traffic_note,
                         "kernel": f"k_scan (variant {last['scan_variant']})", "kernel_ms": statistics.mean(scan_ms),
                         "kernel_share_of_step": statistics.mean(scan_ms) / statistics.mean(step_ms),
                         "ops_per_launch": ops,
                         "ops_model": "SURVEY.md 8(d): 4 INT ops per pre-filter test (tm_stats.tile_tests) + 7 per "
                                      "pair check (6 LOP3 + 1 ISETP, tm_stats.pair_checks), counted by the kernel",
                         "frac_min_ops_model": ops_min / scan_s / 1e12 / ipeak,
                         "min_ops_model": "3 ops per decision (one 64-bit block test: the minimum); DESIGN.md sec. 6",
                         "ncu_same_kernel": ncu, "peak_src": ipeak_src,
                         "build_id": tmx.build_id()},
            "e2e": {"value": e2e_value, "unit": "queries/s", "h2d_bytes_per_step": h2d_bytes,
                    "d2h_bytes_per_step": d2h},
            "gpu_launches": launches,
            "clocks": sampler.summary(),
            "stages_ms": {k: statistics.mean(s[k] for s in stats) for k in
                          ("encode_ms", "route_ms", "scan_ms", "merge_ms", "total_ms")},
            "path_stats": {k: last[k] for k in ("n_partitions", "routed", "candidate_pairs", "tile_tests",
                                                "pair_checks", "matched_sets", "emitted_pairs", "result_pairs",
                                                "work_items", "exact_checked", "exact_kept")},
            "build_s": build_s,
            "memory": mem,
            "tuning_calls": tune_calls,   # untimed calls that finished the variant tuning before the W warm-ups
        }
        if ipeak_raw:
            line["roofline"]["int_peak_microbench"] = {k: ipeak_raw[k] for k in
                                                      ("lop3", "lop3_imad", "precheck_alu", "precheck_imad")
                                                      if k in ipeak_raw}
        if hbm:
            line["hbm"] = hbm
        if ranks:
            line["ranks"] = ranks
        if base:
            line["scaling_base_1gpu"] = base
        if not args.no_cpu_baseline and world == 1:
            from oracle import o2
            ix, q_sig, size, obuild = oracle_rate(wl, c, unique, target_s=args.cpu_s)
            sel = np.sort(np.random.default_rng(1).choice(q_sig.shape[0], size, replace=False))
            t0 = time.perf_counter()
            ix.match(wl.key_off, wl.keys, q_sig[sel], unique, qid=sel.astype(np.uint32))
            dt = time.perf_counter() - t0
            line["cpu_baseline"] = {"value": size / dt, "unit": "queries/s", "cores": o2.threads(0),
                                    "kind": "oracle",
                                    "sample": f"{size} of {Q} queries (" +
                                              (f"O2 brute force over {c['n_sets']} sets, {o2.threads(0)} threads"
                                               if isinstance(ix, _BruteOracle) else
                                               f"O2: Alg.1 MAX_P={c.get('oracle_max_partition')} + Alg.2 + linear scan, "
                                               f"{o2.threads(0)} threads; Alg.1 build {obuild:.1f} s excluded") + ")"}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def finish_tuning(db, step, world, cdev):
    """The handle times its scan-kernel variants on its first calls of a batch size (DESIGN.md
    sec. 6): finish that before the warm-up steps, so that no timed step runs a candidate."""
    import torch
    import torch.distributed as dist
    calls = 0
    for _ in range(16):
        step()
        calls += 1
        done = 0 if db.stats()["tuning"] else 1
        if world > 1:   # the ranks agree (the sharded step has collectives inside)
            t = torch.tensor([done], device=cdev, dtype=torch.int32)
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            done = int(t.item())
        if done:
            break
    return calls


def single_gpu_value(wl, c, args, dev, stream, flush):
    """Scaling base of a sharded N-GPU line: the whole database on rank 0's GPU, the same batch,
    tuning + W warm-ups + K timed steps as the sharded run (device-resident inputs)."""
    import torch
    import paper_conf_eurosys_rogorapkmcc17_b200 as tmb
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=c["max_partition"], device=dev,
                      tile_filter=args.tile_filter, row_order=args.row_order, exact=int(args.exact))
    q = wl.queries
    arrs = [np.ascontiguousarray(a) for a in (q.vocab_bytes, q.vocab_off.view(np.int64),
                                              q.tag_idx.view(np.int32), q.set_off.view(np.int64))]
    dt = [torch.from_numpy(a).to(f"cuda:{dev}") for a in arrs]
    dq = tmb.device_tagsets(dt[0].data_ptr(), dt[1].data_ptr(), dt[2].data_ptr(), dt[3].data_ptr(),
                            arrs[0].size, arrs[1].size - 1, arrs[2].size, q.n_sets)

    def step():
        return db.match_batch_device(dq, bool(args.unique), stream.cuda_stream)

    finish_tuning(db, step, 1, None)
    for _ in range(args.warmup):
        step()
    ms = []
    for _ in range(args.steps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        step()
        b.record(stream)
        b.synchronize()
        ms.append(a.elapsed_time(b))
    st = db.stats()
    db.close()
    return {"value": q.n_sets * len(ms) / (sum(ms) / 1000), "unit": "queries/s", "workload": args.config,
            "ms_per_step": statistics.mean(ms), "scan_ms": st["scan_ms"],
            "note": "the same workload and batch unsharded on rank 0's GPU, same K steps (device-resident inputs)"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=None, help="BASELINE config; default C3 (N = 1), C4 (N > 1)")
    ap.add_argument("--unique", action="store_true", help="match-unique instead of match")
    ap.add_argument("--replicated", action="store_true",
                    help="N > 1: every rank holds the whole database and matches its own batch (weak scaling) "
                         "instead of the default partition sharding + NCCL exchange")
    ap.add_argument("--no-hbm", action="store_true", help="skip the one-partition HBM roofline block")
    ap.add_argument("--no-scaling-base", action="store_true", help="N > 1: skip the 1-GPU base on rank 0")
    # default layout = the B200 one (R18): balanced splits inside partitions +
    # tile AND masks; --tile-filter 0 --row-order 0 is the paper's lexicographic order + Alg. 4 prefix
    ap.add_argument("--tile-filter", type=int, default=1, choices=[0, 1, 2])
    ap.add_argument("--exact", action="store_true",
                    help="exact subset post-check (PAPER.md:106; removes Bloom false positives)")
    ap.add_argument("--row-order", type=int, default=1, choices=[0, 1],
                    help="1: balanced-split order inside partitions (DESIGN.md R18; needs --tile-filter 1)")
    ap.add_argument("--max-partition", type=int, default=-1,
                    help="MAX_P (PAPER.md:361-371 sweep): -1 = auto (TM_AUTO_MAX_PARTITION, default), "
                         "0 = the config's (the paper's 200K), N = N")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-s", type=float, default=10.0, help="seconds of oracle work for cpu_baseline")
    ap.add_argument("--ref-step-s", type=float, default=4.0, help="seconds per --impl reference step")
    args = ap.parse_args()
    if args.config is None:
        args.config = "C3" if int(os.environ.get("WORLD_SIZE", "1")) == 1 else "C4"
    if args.warmup < 3:
        args.warmup = 3
    if args.row_order == 1 and args.tile_filter == 0:
        args.row_order = 0   # the first/last prefix needs lexicographic order
    load_workload.max_partition = args.max_partition
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
