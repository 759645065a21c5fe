"""Summarise an ncu --set full report of the scan kernel (run here, no GPU needed).

usage: python scripts/ncu_summary.py gpurun_out/<tag>_scan.ncu-rep [--config C2] [--json profiles/x.json]
Prints the metrics the roofline needs (duration, DRAM bytes, ALU / issue
utilisation, occupancy, L2 hit rate, shared-memory conflicts) and the top warp
stall reasons.
"""
import csv
import io
import json
import subprocess
import sys

NCU = "/usr/local/cuda/bin/ncu"
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.per_cycle_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_registers",
    "launch__shared_mem_per_block_static", "lts__t_sector_hit_rate.pct",
    "sm__cycles_elapsed.avg.per_second", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__inst_executed_op_global_atom.sum", "smsp__inst_executed_op_global_red.sum",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
]


def load(path):
    out = subprocess.run([NCU, "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [dict(zip(hdr, r)) for r in rows[2:]], dict(zip(hdr, units))


def num(v):
    try:
        return float(str(v).replace(",", ""))
    except Exception:
        return None


def main():
    path = sys.argv[1]
    cfg = sys.argv[sys.argv.index("--config") + 1] if "--config" in sys.argv else "C2"
    launches, units = load(path)
    lines = []
    for i, m in enumerate(launches):
        lines.append(f"== launch {i}: {m.get('Kernel Name', '')[:80]}")
        for k in KEYS:
            if k in m:
                lines.append(f"  {k:66s} {m[k]:>18s} {units.get(k, '')}")
        st = []
        for k, v in m.items():
            for pre, suf in (("smsp__average_warp_latency_issue_stalled_", ".ratio"),
                             ("smsp__average_warps_issue_stalled_", "_per_issue_active.ratio")):
                if k.startswith(pre) and k.endswith(suf):
                    x = num(v)
                    if x:
                        st.append((x, k[len(pre):-len(suf)]))
        lines.append("  top stall reasons (avg cycles per issued instruction):")
        for x, k in sorted(st, reverse=True)[:10]:
            lines.append(f"    {k:40s} {x:8.2f}")
    text = "\n".join(lines)
    print(text)
    if "--json" in sys.argv:
        m = launches[0]
        rd, wr = num(m.get("dram__bytes_read.sum")), num(m.get("dram__bytes_write.sum"))
        # ncu reports bytes in the unit given in the units row
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rs = scale.get(units.get("dram__bytes_read.sum", "byte"), 1)
        ws = scale.get(units.get("dram__bytes_write.sum", "byte"), 1)
        js = {"config": cfg, "report": path, "kernel": m.get("Kernel Name", ""),
              "dram_bytes_per_launch": (rd or 0) * rs + (wr or 0) * ws,
              "duration_ns": num(m.get("gpu__time_duration.sum")),
              "duration_unit": units.get("gpu__time_duration.sum"),
              "alu_pipe_pct": num(m.get("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active")),
              "issue_active_pct": num(m.get("smsp__issue_active.avg.pct_of_peak_sustained_active")),
              "warps_active_pct": num(m.get("sm__warps_active.avg.pct_of_peak_sustained_active")),
              "l2_hit_pct": num(m.get("lts__t_sector_hit_rate.pct")),
              # the library build and scan variant the capture was taken on (bench.py only uses the
              # traffic for a line of the same build and variant)
              "build_id": sys.argv[sys.argv.index("--build-id") + 1] if "--build-id" in sys.argv else None,
              "variant": int(sys.argv[sys.argv.index("--variant") + 1]) if "--variant" in sys.argv else None}
        with open(sys.argv[sys.argv.index("--json") + 1], "w") as f:
            json.dump(js, f, indent=1)


if __name__ == "__main__":
    main()
