"""Time the GPU minimum cycle basis (ear_mcb, paper sec. 3) on the configs' graphs.

    python tools/time_mcb.py [cfg1 cfg2 ...] [--out profiles/...jsonl]
Prints one JSON line per config: device time of one ear_mcb call after a warm-up call, MCB weight,
dimension, reduced sizes, candidate count.  (Parity: tests/test_mcb_gpu.py.)
"""
import argparse
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["cfg1", "cfg2"])
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    lines = []
    for name in args.configs:
        g = gg.config(name)
        src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
        ea.mcb(g.n, src, dst, w).destroy()   # warm-up
        torch.cuda.synchronize()
        t = time.perf_counter()
        r = ea.mcb(g.n, src, dst, w)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t
        info = r.info()
        r.destroy()
        rec = {"config": name, "n": g.n, "m": g.m, "seconds": dt, **info,
               "phases_per_s": info["dim"] / dt if dt > 0 else None}
        print(json.dumps(rec), flush=True)
        lines.append(rec)
    if args.out:
        with open(args.out, "w") as f:
            for r in lines:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
