"""Quick look at one kernel in an ncu report: key throughput metrics, stall reasons, hottest SASS lines
and the executed-instruction mix by loop body.   python tools/ncu_quick.py <rep> [n_hot]"""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
nhot = int(sys.argv[2]) if len(sys.argv) > 2 else 15


def ncu(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout


rows = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv", "--print-units", "base"))))
hdr, d = rows[0], rows[2]
want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "smsp__inst_executed.sum", "launch__occupancy_limit_shared_mem",
        "launch__occupancy_limit_registers", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct"]
for w in want:
    if w in hdr:
        print(f"  {w:70s} {d[hdr.index(w)]}")
st = [(h[len("smsp__average_warps_issue_stalled_"):].split("_per_issue_active")[0], d[i]) for i, h in enumerate(hdr)
      if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio")]
st = sorted([(float(v), k) for k, v in st if v], reverse=True)[:8]
print("  stalls:", ", ".join(f"{k} {v:.2f}" for v, k in st))
rows = list(csv.reader(io.StringIO(ncu("--page", "source", "--csv", "--print-source", "sass"))))
hdr, data = rows[1], rows[2:]
si, src, ex = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source"), hdr.index("Instructions Executed")
tot = sum(int(r[si]) for r in data if r[si].isdigit()) or 1
for i in sorted(range(len(data)), key=lambda i: -int(data[i][si]) if data[i][si].isdigit() else 0)[:nhot]:
    r = data[i]
    print(f"  {i:5d} {int(r[si]) / tot * 100:5.1f}% ex={r[ex]:>10} {r[src][:90]}")
agg = collections.Counter()
for r in data:
    if r[ex].isdigit():
        agg[int(r[ex])] += 1
t = sum(k * v for k, v in agg.items()) or 1
print("  instruction mix by execution count (count x #instructions):")
for k, v in sorted(agg.items(), key=lambda kv: -kv[0] * kv[1])[:8]:
    print(f"    {k:>10} x {v:4d}  {k * v / t * 100:5.1f}%")
