#!/usr/bin/env python
"""bench.py -- TagMatch B200 throughput (driver contract).

A step = one tm_match_batch over one batch of queries = the whole hot path
(encode, route, batch, pre-filter, subset scan, compaction,
key expansion, sort/merge).  Default workload: BASELINE config C2 (1M tag
sets, 100k-query stream, MAX_P = 200K), `match` (Table 1).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C2] [--unique]

value  : queries/s over all ranks, inputs resident in HBM (tm_match_batch_device),
         per-step CUDA events on the launching stream, L2 flushed between steps.
e2e    : queries/s through tm_match_batch_csr with pinned host queries (H2D inside
         the timed region) and the result -- every query's sorted keys -- copied
         back to host (D2H: 4 B per pair + 8 B per query offset).
N > 1  : one process per GPU (torchrun); every rank holds a replica of the
         database and matches its own query batch (replicated mode, PAPER.md:110,
         228: no data-path collective) -> "scaling": "weak"; time = max over ranks.
         --shard: the database is partition-sharded over the ranks, every
         rank matches the same batch against its partitions and the pairs go to
         query owners over NCCL (tm_match_batch_sharded_device) -> "strong".
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
ALU_LANES_PER_SM_CLK = 64     # LOP3/IADD3 ALU pipe: 16 lanes/clk/SMSP x 4 SMSP (B300_MICROARCH.md)
SM_COUNT = 148
# algorithmic INT ops per decision: every pre-filter test
# (mask vs query) and every pair check (set vs query) needs at least one 64-bit
# block test = and-not of both 32-bit halves + zero test = 3 ALU ops.
OPS_PER_TILE_TEST = 3
OPS_PER_PAIR_CHECK = 3
SURVEY_OPS_PER_TILE_TEST = 4    # SURVEY.md 8(d) per-unit figures (plain Alg. 4 / Alg. 3)
SURVEY_OPS_PER_PAIR_CHECK = 7


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
        c = dict(tmgen.CRAFTED[name], max_partition=getattr(load_workload, "max_partition", 0) or 200_000, total_tags=0)
        wl = tmgen.config(name, max_partition=c["max_partition"],
                          query_seed=c["seed"] + (1 << 32) + 7919 * rank)
        return wl, c
    c = dict(tmgen.CONFIGS[name])
    if getattr(load_workload, "max_partition", 0):
        c["max_partition"] = load_workload.max_partition
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
        ix = o2.Index(db_sig, c["max_partition"])
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
            "config": config_block(c, args, wl),
            "cpu_baseline": {"value": value, "unit": "queries/s", "cores": cores, "kind": "oracle",
                             "sample": f"{size} of {q_sig.shape[0]} queries per step ("
                                       + (f"O2 brute force over {c['n_sets']} sets" if isinstance(ix, _BruteOracle)
                                          else f"O2: Alg.1 MAX_P={c['max_partition']} + Alg.2 + linear scan; "
                                               f"Alg.1 build {build_s:.1f} s excluded") + ")"},
            "e2e": {"value": value, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_block(c, args, wl):
    return {"workload": args.config, "n_sets": c["n_sets"], "n_queries": c["n_queries"],
            "query_tags": (f"{c['set_tags']}-tag DB sets, {c['query_tags']}-tag queries (PAPER.md:391-399)"
                           if "set_tags" in c else
                           "base set + 2..4 extra" if not c["total_tags"] else f"total {c['total_tags']}"),
            "max_partition": c["max_partition"], "mode": "match-unique" if args.unique else "match",
            "tile_filter": ["alg4-prefix", "tile-and", "none"][args.tile_filter],
            "row_order": ["lexicographic", "balanced-splits"][args.row_order],
            "exact_check": bool(args.exact),
            "parallelism": (f"partition-sharded-{args.gpus} (NCCL exchange)" if args.shard else
                            f"replicated-dp{args.gpus}") if args.gpus > 1 else "single",
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
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(pg)
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()

    import __graft_entry__
    __graft_entry__.build() if rank == 0 or world == 1 else None
    if world > 1:
        dist.barrier()
    import paper_conf_eurosys_rogorapkmcc17_b200 as tmb

    sharded = args.shard and world > 1
    # replicated mode: every rank its own batch; sharded mode: the same batch on every rank
    wl, c = load_workload(args.config, 0 if sharded else rank)
    unique = bool(args.unique)
    Q = wl.queries.n_sets
    torch.cuda.synchronize(dev)
    mem0 = (torch.cuda.mem_get_info(dev)[0], torch.cuda.memory_reserved(dev))
    t0 = time.perf_counter()
    db = tmb.Database(wl.db, wl.key_off, wl.keys, max_partition=c["max_partition"], device=dev,
                      tile_filter=args.tile_filter, row_order=args.row_order, exact=int(args.exact),
                      n_shards=world if sharded else 1, shard=rank if sharded else 0)
    build_s = time.perf_counter() - t0
    torch.cuda.synchronize(dev)
    mem1 = (torch.cuda.mem_get_info(dev)[0], torch.cuda.memory_reserved(dev))
    if sharded:
        from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as tmx
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
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=f"cuda:{dev}")
    stream = torch.cuda.current_stream()

    def step_device():
        if sharded:
            return db.match_batch_sharded_device(dq, unique, stream.cuda_stream)
        return db.match_batch_device(dq, unique, stream.cuda_stream)

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

    # the handle times its scan-kernel variants on its first calls of a batch size (DESIGN.md
    # sec. 6): finish that before the W warm-up steps, so that no timed step runs a candidate
    tune_calls = 0
    for _ in range(16):
        step_device()
        tune_calls += 1
        done = 0 if db.stats()["tuning"] else 1
        if world > 1:   # the ranks agree (the sharded step has collectives inside)
            t = torch.tensor([done], device=f"cuda:{dev}" if pg == "nccl" else "cpu", dtype=torch.int32)
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            done = int(t.item())
        if done:
            break
    for _ in range(args.warmup):
        step_device()
        step_e2e()
    torch.cuda.synchronize()

    # ---- value: device-resident inputs, per-step CUDA events, L2 flushed between steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    launches, scan_ms, stats = 0, [], []
    sampler = ClockSampler(dev)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with sampler:
        for i in range(args.steps):
            flush.zero_()
            ev[i][0].record(stream)
            out = step_device()
            ev[i][1].record(stream)
            st = db.stats()
            launches += st["kernel_launches"]
            scan_ms.append(st["scan_ms"])
            stats.append(st)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    t_local = sum(step_ms) / 1000.0
    t_max = t_local
    if world > 1:
        t = torch.tensor([t_local], device=f"cuda:{dev}" if pg == "nccl" else "cpu", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t_max = float(t.item())
    value = (1 if sharded else world) * Q * args.steps / t_max

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
        t = torch.tensor([e2e_local], device=f"cuda:{dev}" if pg == "nccl" else "cpu", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_local = float(t.item())
    e2e_value = (1 if sharded else world) * Q * args.steps / e2e_local

    if rank == 0:
        peaks, peak_src = measured_peaks()
        last = stats[-1]
        ops = OPS_PER_TILE_TEST * last["tile_tests"] + OPS_PER_PAIR_CHECK * last["pair_checks"]
        scan_s = statistics.mean(scan_ms) / 1000.0
        peak_tops = SM_COUNT * ALU_LANES_PER_SM_CLK * peaks.get("sm_max_mhz", 1965.0) * 1e6 / 1e12
        achieved = ops / scan_s / 1e12
        traffic, ncu = None, None
        try:
            per_cfg = os.path.join(ROOT, "profiles", f"ncu_scan_traffic_{args.config}.json")
            with open(per_cfg if os.path.exists(per_cfg) else
                      os.path.join(ROOT, "profiles", "ncu_scan_traffic.json")) as f:
                tr = json.load(f)
                if tr.get("config") == args.config:
                    traffic = tr.get("dram_bytes_per_launch")
                    ncu = {k: tr.get(k) for k in ("alu_pipe_pct", "issue_active_pct", "warps_active_pct",
                                                  "l2_hit_pct")}
                    ncu["report"] = tr.get("report")
        except Exception:
            pass
        line = {
            "metric": METRIC, "value": value, "unit": "queries/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": statistics.mean(step_ms), "higher_is_better": True,
            "scaling": "strong" if sharded else "weak", "vs_baseline": None, "dtype": "u64",
            "data": ("synthetic (seeded sec. 4.4 crafted workload, tmgen.generate_crafted, PAPER.md:391-399)"
                     if args.config.startswith(("C6", "C7")) else
                     "synthetic (seeded Twitter-like generator tmgen, PAPER.md:258-282)"),
            "config": config_block(c, args, wl),
            "roofline": {"bound": "alu", "achieved": achieved, "peak": peak_tops, "unit": "Tops/s",
                         "frac": achieved / peak_tops, "traffic": traffic,
                         "kernel": f"k_scan (variant {last['scan_variant']})", "kernel_ms": statistics.mean(scan_ms),
                         "kernel_share_of_step": statistics.mean(scan_ms) / statistics.mean(step_ms),
                         "ops_per_launch": ops,
                         "ops_model": "3 ALU ops per decision (pre-filter test or pair check): the minimum "
                                      "one 64-bit block test; DESIGN.md sec. 6",
                         "frac_survey_model": (SURVEY_OPS_PER_TILE_TEST * last["tile_tests"] +
                                               SURVEY_OPS_PER_PAIR_CHECK * last["pair_checks"]) / scan_s / 1e12
                                              / peak_tops,
                         "survey_model": "SURVEY.md 8(d): 4 ops per tile test + 7 per pair check (the full "
                                         "three-block check); informational, frac above is the primary",
                         "ncu_same_kernel": ncu,
                         "peak_src": f"{SM_COUNT} SMs x {ALU_LANES_PER_SM_CLK} ALU lanes/clk x "
                                     f"{peaks.get('sm_max_mhz', 1965.0)} MHz ({peak_src} sm_max_mhz)"},
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
            "memory": memory_block(db, mem0, mem1, dev),
            "tuning_calls": tune_calls,   # untimed calls that finished the variant tuning before the W warm-ups
        }
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
                                               f"O2: Alg.1 MAX_P={c['max_partition']} + Alg.2 + linear scan, "
                                               f"{o2.threads(0)} threads; Alg.1 build {obuild:.1f} s excluded") + ")"}
        print(json.dumps(line), flush=True)
    db.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--unique", action="store_true", help="match-unique instead of match")
    ap.add_argument("--shard", action="store_true",
                    help="N > 1: partition-sharded database + NCCL exchange (strong scaling) instead of replicas")
    # default layout = the B200 one (R18): balanced splits inside partitions +
    # tile AND masks; --tile-filter 0 --row-order 0 is the paper's lexicographic order + Alg. 4 prefix
    ap.add_argument("--tile-filter", type=int, default=1, choices=[0, 1, 2])
    ap.add_argument("--exact", action="store_true",
                    help="exact subset post-check (PAPER.md:106; removes Bloom false positives)")
    ap.add_argument("--row-order", type=int, default=1, choices=[0, 1],
                    help="1: balanced-split order inside partitions (DESIGN.md R18; needs --tile-filter 1)")
    ap.add_argument("--max-partition", type=int, default=0,
                    help="override the config's MAX_P (PAPER.md:361-371 sweep); 0 = config value")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-s", type=float, default=10.0, help="seconds of oracle work for cpu_baseline")
    ap.add_argument("--ref-step-s", type=float, default=8.0, help="seconds per --impl reference step")
    args = ap.parse_args()
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
