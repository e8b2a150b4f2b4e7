#!/usr/bin/env python
"""Summarise ncu outputs brought back in gpurun_out/ into tracked files under profiles/.

    python tools/ncu_summary.py launches <launches.csv> <out.txt>
    python tools/ncu_summary.py report <prof.ncu-rep> <out.txt> [--traffic-key WORKLOAD:KERNEL] [--launch i]

`launches`: per-kernel launch count, summed device time and share of the captured step
(cold-cache, serialised ncu timings: compare shares, not absolutes).
`report`: the key metrics of an `ncu --set full` capture (duration, DRAM bytes, pipe utilisation,
occupancy, stall reasons); with --traffic-key it also records dram_bytes_per_launch into
profiles/ncu_traffic.json, which bench.py reads for roofline.traffic.
"""
import collections
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = ["Kernel Name", "Grid Size", "Block Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__warps_eligible.avg.per_cycle_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "launch__waves_per_multiprocessor",
        "sm__cycles_elapsed.avg.per_second", "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "smsp__inst_executed.sum"]


def to_ms(v, unit):
    return v / {"ns": 1e6, "nsecond": 1e6, "us": 1e3, "usecond": 1e3, "ms": 1.0, "msecond": 1.0}.get(unit, 1.0)


def launches(path, out):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr, data = rows[h], rows[h + 1:]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in data:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0]
        agg[name][0] += 1
        agg[name][1] += to_ms(float(r[vi].replace(",", "")), r[ui])
    tot = sum(v[1] for v in agg.values())
    lines = [f"# ncu launch list: {os.path.basename(path)}  (gpu__time_duration.sum, --clock-control none;",
             "#  cold-cache serialised replay: compare shares, not absolute times)",
             f"# total {tot:.3f} ms over {sum(v[0] for v in agg.values())} launches", "",
             f"{'kernel':70s} {'launches':>8s} {'ms':>11s} {'share':>8s}"]
    for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"{k[:70]:70s} {c:8d} {t:11.3f} {100 * t / tot:7.2f}%")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:12]))


def report(path, out, traffic_key=None, launch_idx=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units, data = rows[0], rows[1], rows[2:]
    lines = [f"# ncu --set full summary: {os.path.basename(path)}", ""]
    per_launch = []
    for li, d in enumerate(data):
        lines.append(f"## launch {li}")
        rec = {}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                lines.append(f"  {k:72s} {d[i]:>24s} {units[i]}")
                rec[k] = (d[i], units[i])
        stalls = []
        for i, name in enumerate(hdr):
            if "average_warps_issue_stalled" in name and name.endswith("per_issue_active.ratio"):
                try:
                    v = float(d[i])
                except ValueError:
                    continue
                if v >= 0.05:
                    stalls.append((v, name.replace("smsp__average_warps_issue_stalled_", "").replace(
                        "_per_issue_active.ratio", "")))
        lines.append("  stalls (warps per issue-active cycle): " +
                     ", ".join(f"{n} {v:.2f}" for v, n in sorted(stalls, reverse=True)))
        lines.append("")
        per_launch.append(rec)
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))
    if traffic_key:
        wl, kern = traffic_key.split(":")
        idx = launch_idx if launch_idx is not None else len(per_launch) - 1
        rec = per_launch[idx]

        def gb(k):
            v, u = rec[k]
            return float(v) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}.get(u, 1.0)

        tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        t = json.load(open(tpath)) if os.path.exists(tpath) else {}
        t.setdefault(wl, {})[kern] = {"dram_bytes_per_launch": gb("dram__bytes_read.sum") + gb("dram__bytes_write.sum"),
                                      "source": os.path.relpath(out, ROOT), "launch": idx,
                                      "grid": rec.get("Grid Size", ("", ""))[0]}
        json.dump(t, open(tpath, "w"), indent=1)


if __name__ == "__main__":
    cmd = sys.argv[1]
    if cmd == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        tk = None
        li = None
        if "--traffic-key" in sys.argv:
            tk = sys.argv[sys.argv.index("--traffic-key") + 1]
        if "--launch" in sys.argv:
            li = int(sys.argv[sys.argv.index("--launch") + 1])
        report(sys.argv[2], sys.argv[3], tk, li)
