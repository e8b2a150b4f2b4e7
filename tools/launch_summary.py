"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list into kernel | launches | ms | share.

    python tools/launch_summary.py gpurun_out/launches.csv "description" > profiles/....txt
"""
import collections
import csv
import sys

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3}


def main():
    path, desc = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
    hdr, agg = None, collections.defaultdict(lambda: [0, 0.0])
    for r in csv.reader(open(path)):
        if r and r[0] == "ID":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d["Metric Name"] != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"].split("(")[0].replace("(anonymous namespace)::", "").replace("<unnamed>::", "")
        agg[name][0] += 1
        agg[name][1] += float(d["Metric Value"].replace(",", "")) * SCALE[d["Metric Unit"]]
    tot = sum(v[1] for v in agg.values())
    print(f"# {desc}")
    print("# gpu__time_duration.sum per launch (ncu --clock-control none: cold-cache, serialised); share of the summed time")
    print(f"# launches {sum(v[0] for v in agg.values())}, summed kernel time {tot:.2f} ms")
    print("kernel | launches | total ms | share")
    for k, (c, ms) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{k} | {c} | {ms:.3f} | {100 * ms / tot:.2f}%")


if __name__ == "__main__":
    main()
