#!/usr/bin/env python
"""cfg3 (BASELINE.json configs[2]): 50k-vertex tori with degree-two fraction f = 0/20/40/60/80 %,
ear-reduced APSP (plain FW and Phase II by blocks) vs direct blocked FW on the whole graph
(EAR_FLAG_NO_CONTRACT), one B200.

For every f: one warm-up + one timed apsp_full per variant (CUDA events), the two 10 GB outputs
compared bit for bit on the device (pin P7), and the FW min-plus rate.  Prints one JSON line per f
and writes them to the path given by --out.
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


def timed(fn):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    torch.cuda.synchronize()
    ea.profile_reset()
    ea.profile_enable(True)
    e0.record()
    fn()
    e1.record()
    torch.cuda.synchronize()
    prof = ea.profile_read()
    ea.profile_enable(False)
    return e0.elapsed_time(e1), prof


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--fs", default="0,20,40,60,80")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    lines = []
    for f in [int(x) for x in args.fs.split(",")]:
        g = gg.config(f"cfg3_f{f}")
        st = gg.stats(g)
        src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
        out_r = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
        plan = ea.ear_decompose(g.n, src, dst, w)
        nr = plan.info().n_reduced
        plan.destroy()
        ms_r, pr = timed(lambda: ea.apsp_full(g.n, src, dst, w, out=out_r))
        out_d = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
        ms_d, pd = timed(lambda: ea.apsp_full(g.n, src, dst, w, out=out_d, flags=ea.FLAG_NO_CONTRACT))
        same = bool(torch.equal(out_r, out_d))
        del out_d
        out_b = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
        ms_b, _ = timed(lambda: ea.apsp_full(g.n, src, dst, w, out=out_b, flags=ea.FLAG_BCC))
        same_b = bool(torch.equal(out_r, out_b))
        del out_r, out_b
        torch.cuda.empty_cache()
        rec = {"config": f"cfg3_f{f}", "n": g.n, "m": g.m, "deg2_frac": st["deg2_frac"], "n_reduced": nr,
               "ear_reduced_ms": ms_r, "direct_fw_ms": ms_d, "speedup": ms_d / ms_r,
               "ear_entries_per_s": g.n * g.n / (ms_r / 1e3), "direct_entries_per_s": g.n * g.n / (ms_d / 1e3),
               "ear_fw_phase3_tminplus": pr["fw_phase3_minplus"] / (pr["fw_phase3_ms"] / 1e3) / 1e12,
               "direct_fw_phase3_tminplus": pd["fw_phase3_minplus"] / (pd["fw_phase3_ms"] / 1e3) / 1e12,
               "ear_expand_ms": pr["expand_ms"], "bitwise_equal": same,
               "ear_bcc_ms": ms_b, "bcc_speedup": ms_d / ms_b, "bcc_bitwise_equal": same_b}
        print(json.dumps(rec), flush=True)
        lines.append(rec)
    if args.out:
        with open(args.out, "w") as fh:
            for r in lines:
                fh.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
