"""Per-source-line instruction counts and stall samples of one kernel from an ncu SASS source page.

    python tools/sass_lines.py <ncu sass.csv> <object .o with -lineinfo> <kernel-substring> [--top 40]

The ncu page (`ncu -i X.ncu-rep --page source --csv --print-source sass`) carries per-SASS-address
`Instructions Executed` and stall samples; nvdisasm --print-line-info on the SAME object maps each
function offset to the file:line it came from (inlined headers included).  The object must be the one
that was profiled (rebuild before profiling, not after)."""
import argparse
import collections
import csv
import os
import re
import subprocess
import tempfile


def line_map(obj, ksub):
    with tempfile.TemporaryDirectory() as d:
        subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, check=True,
                       stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
        cubin = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
        txt = subprocess.run(["nvdisasm", "--print-line-info", "-c", os.path.join(d, cubin)], check=True,
                             capture_output=True, text=True).stdout.split("\n")
    out, cur, inside, name = {}, None, False, None
    for ln in txt:
        if re.match(r"^_Z\S+:$", ln):
            inside = ksub in ln
            name = ln[:-1] if inside else name
            continue
        if not inside:
            continue
        if ln.startswith("//----") or ln.startswith(".L_x") and ln.endswith(":") and "(" in ln:
            continue
        m = re.search(r'## File "([^"]+)", line (\d+)', ln)
        if m:
            cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m = re.search(r"/\*([0-9a-f]{4,})\*/", ln)
        if m and cur:
            out.setdefault(int(m.group(1), 16), cur)
    return out, name


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("obj")
    ap.add_argument("kernel")
    ap.add_argument("--top", type=int, default=40)
    a = ap.parse_args()
    off2line, name = line_map(a.obj, a.kernel)
    rows = list(csv.reader(open(a.csv)))
    hdr = next(i for i, r in enumerate(rows) if "Source" in r and any("Instructions Executed" in c for c in r))
    h = rows[hdr]
    ie, ad = h.index("Instructions Executed"), h.index("Address")
    ss = h.index("Warp Stall Sampling (All Samples)")
    data = [(int(r[ad], 16), float(r[ie] or 0), float(r[ss] or 0)) for r in rows[hdr + 1:]
            if len(r) >= len(h) and r[ad].startswith("0x")]
    base = min(x[0] for x in data)
    agg = collections.defaultdict(lambda: [0.0, 0.0])
    for addr, n, s in data:
        agg[off2line.get(addr - base, ("?", 0))][0] += n
        agg[off2line.get(addr - base, ("?", 0))][1] += s
    ti = sum(v[0] for v in agg.values()) or 1.0
    ts = sum(v[1] for v in agg.values()) or 1.0
    srcs = {}
    print(f"# {name}\n# {len(data)} SASS instructions, {ti:.4g} warp-instructions executed")
    for (f, ln), (n, s) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:a.top]:
        if f not in srcs:
            path = os.path.join(os.path.dirname(a.obj), "..", "csrc", f)
            srcs[f] = open(path).read().split("\n") if os.path.exists(path) else []
        text = srcs[f][ln - 1].strip()[:90] if 0 < ln <= len(srcs[f]) else ""
        print(f"inst {100 * n / ti:5.1f}%  stall {100 * s / ts:5.1f}%  {f}:{ln}  {text}")


if __name__ == "__main__":
    main()
