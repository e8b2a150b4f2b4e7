#!/usr/bin/env python
"""Phase II routes side by side on the BASELINE.json configs (one B200): the region route (EAR_FLAG_PART,
the bench's), blocks + per-source SSSP (FLAG_BCC | FLAG_SSSP) and, where it is affordable, blocks + FW.

Per config: Phase II alone (apsp_reduced into the int32 D of G^r; one warm-up call, then one timed call,
CUDA events) for every route with the D matrices compared bit for bit on the device, and the full APSP
(apsp_full, N x N int32 output) for the region route and blocks + SSSP when the output fits beside it
(cfg5's 160 GB does not: Phase II only).  The region route's partition statistics are recorded.
One JSON line per config on stdout and in --out.

    python tools/time_routes.py [--configs cfg1,cfg2,cfg3_f0,...] [--out file.jsonl]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402

ROUTES = {"part": ea.FLAG_PART, "bcc_sssp": ea.FLAG_BCC | ea.FLAG_SSSP, "bcc_fw": ea.FLAG_BCC}


def timed(fn):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="cfg1,cfg2,cfg3_f0,cfg3_f20,cfg3_f40,cfg3_f60,cfg3_f80,cfg4,cfg5")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    for name in args.configs.split(","):
        g = gg.config(name)
        src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
        rec = {"config": name, "n": g.n, "m": g.m}
        Ds = {}
        for r, fl in ROUTES.items():
            if r == "bcc_fw" and name in ("cfg3_f0", "cfg3_f20", "cfg5"):
                continue   # seconds per call: covered by earlier sweeps
            p = ea.ear_decompose(g.n, src, dst, w, flags=fl)
            rec["n_reduced"] = p.info().n_reduced
            if r == "part":
                rec["part"] = p.part_info()
            D = ea.alloc_D(p)
            rec[f"phase2_{r}_ms"] = timed(lambda: ea.apsp_reduced(p, D))
            Ds[r] = D
            p.destroy()
        base = Ds["part"]
        rec["phase2_D_equal"] = all(torch.equal(base, D) for D in Ds.values())
        del Ds, base, D
        torch.cuda.empty_cache()
        free = torch.cuda.mem_get_info()[0]
        if 2.2 * 4.0 * g.n * g.n < free:
            outs = {}
            for r in ("part", "bcc_sssp"):
                out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
                rec[f"full_{r}_ms"] = timed(lambda: ea.apsp_full(g.n, src, dst, w, out=out, flags=ROUTES[r]))
                rec[f"full_{r}_entries_per_s"] = g.n * g.n / (rec[f"full_{r}_ms"] / 1e3)
                outs[r] = out
            rec["full_equal"] = torch.equal(outs["part"], outs["bcc_sssp"])
            del outs, out
            torch.cuda.empty_cache()
        line = json.dumps(rec)
        print(line, flush=True)
        if args.out:
            with open(args.out, "a") as f:
                f.write(line + "\n")


if __name__ == "__main__":
    main()
