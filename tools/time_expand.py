"""Expansion A/B on a config and labelling: the pair-major kernel (default) against the row-group kernel
(EAR_EXPAND_PAIRS=0) on the same D (Phase II by blocks), outputs compared entry for entry, device time
per expand_ears call (5 after 2 warm-ups) with the library's per-kernel profile (k_expand_pairs alone,
the u16 narrowing of D apart).

    python tools/time_expand.py [cfg4] [--labels morton|random] [--out file.jsonl]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="cfg4")
    ap.add_argument("--labels", default="morton")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    g = gg.config(args.config, 0, args.labels)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_BCC)
    D = ea.alloc_D(plan)
    ea.apsp_reduced(plan, D)
    nr = plan.info().n_reduced
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    outs, lines = {}, []
    for mode in ("rowgroup", "pairs"):
        os.environ["EAR_EXPAND_PAIRS"] = "0" if mode == "rowgroup" else "1"
        out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
        for _ in range(2):
            ea.expand_ears(plan, D, 0, g.n, out=out)
        torch.cuda.synchronize()
        ea.profile_reset()
        ea.profile_enable(True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(5):
            ea.expand_ears(plan, D, 0, g.n, out=out)
        e1.record()
        torch.cuda.synchronize()
        p = ea.profile_read()
        ea.profile_enable(False)
        ms = e0.elapsed_time(e1) / 5
        alg = 4.0 * g.n * g.n + 4.0 * nr * nr + 16.0 * g.n
        kms = p["expand_ms"] / 5
        rec = {"config": args.config, "labels": args.labels, "kernel": mode, "n": g.n, "n_reduced": nr,
               "call_ms": ms, "kernel_ms": kms, "d16_ms": p["expand_d16_ms"] / 5, "same_chain_ms": p["same_chain_ms"] / 5,
               "algorithmic_GB": alg / 1e9, "kernel_GBps": alg / (kms / 1e3) / 1e9,
               "kernel_frac_of_copy_bw": alg / (kms / 1e3) / 1e9 / peaks["hbm_gbs"],
               "call_frac_of_copy_bw": alg / (ms / 1e3) / 1e9 / peaks["hbm_gbs"]}
        outs[mode] = out
        lines.append(rec)
    os.environ.pop("EAR_EXPAND_PAIRS", None)
    same = bool(torch.equal(outs["rowgroup"], outs["pairs"]))
    for r in lines:
        r["outputs_identical"] = same
        print(json.dumps(r), flush=True)
    if args.out:
        with open(args.out, "a") as f:
            for r in lines:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
