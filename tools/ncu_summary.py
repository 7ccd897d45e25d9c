"""Summarise an ncu --set full report into profiles/ (run here, no GPU needed).

usage: python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/<name>.md [workload]
Writes a markdown summary; with a workload name also records the dominant
kernel's DRAM bytes per launch in profiles/ncu_traffic.json (read by bench.py).
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("lts__t_sectors.sum", "L2 sectors"),
    ("lts__t_sectors_op_atom.sum", "L2 atomic sectors"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput %"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "global load sectors"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "global load requests"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "warp execution efficiency (threads/inst)"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__cluster_dim_x", "cluster"),
]


def main():
    rep, out = sys.argv[1], sys.argv[2]
    workload = sys.argv[3] if len(sys.argv) > 3 else None
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    lines = [f"# ncu summary: {os.path.basename(rep)}", ""]
    traffic = None
    total = 0.0  # summed over every captured launch (e.g. the select kernel of each hop of one step)
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        lines.append(f"## {name}")
        lines.append("")
        lines.append("| metric | value | unit |")
        lines.append("|---|---|---|")
        vals = {}
        for k, label in KEYS:
            if k in hdr:
                i = hdr.index(k)
                vals[k] = r[i]
                lines.append(f"| {label} (`{k}`) | {r[i]} | {units[i]} |")
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued"):
                try:
                    stalls.append((float(r[i]), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        tot = sum(s for s, _ in stalls) or 1.0
        lines.append("")
        lines.append("Top stall reasons (PC sampling): " +
                     ", ".join(f"{n} {100 * s / tot:.1f}%" for s, n in stalls[:6]))
        lines.append("")
        try:
            def gb(key):
                i = hdr.index(key)
                v = float(r[i])
                return v * {"Tbyte": 1e12, "Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}.get(units[i], 1.0)
            traffic = gb("dram__bytes_read.sum") + gb("dram__bytes_write.sum")
            total += traffic
            lines.append(f"DRAM bytes (read + write) per launch: {traffic:.4g}")
            lines.append("")
        except (ValueError, KeyError):
            pass
    if len(rows) > 3:
        lines.append(f"DRAM bytes (read + write) summed over the {len(rows) - 2} captured launches: {total:.4g}")
        traffic = total
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    if workload and traffic is not None:
        path = os.path.join(os.path.dirname(out), "ncu_traffic.json")
        d = {}
        if os.path.exists(path):
            d = json.load(open(path))
        d[workload] = traffic
        json.dump(d, open(path, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
