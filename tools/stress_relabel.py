"""Random-relabel stress rows: the same generators with a seeded random permutation of the
vertex ids instead of the spatially coherent Morton labelling -- the expansion's worst case (3.4 D-row
gathers per output against 0.85).  Per config and labelling: one apsp_full step (bench flags, after a
warm-up), its expansion kernel time and algorithmic GB/s from the library's profile.  Parity with random
labels: tests/test_parity_gpu.py (test_cfg2_random_relabel_full and the quarter-size cfg4 one).

    python tools/stress_relabel.py [cfg2 cfg4] [--out profiles/...jsonl]
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
    ap.add_argument("configs", nargs="*", default=["cfg2", "cfg4"])
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    lines = []
    for name in args.configs:
        for labels in ("morton", "random"):
            g = gg.config(name, 0, labels)
            src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
            out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
            ea.apsp_full(g.n, src, dst, w, out=out, flags=ea.FLAG_BCC)
            torch.cuda.synchronize()
            ea.profile_reset()
            ea.profile_enable(True)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ea.apsp_full(g.n, src, dst, w, out=out, flags=ea.FLAG_BCC)
            e1.record()
            torch.cuda.synchronize()
            p = ea.profile_read()
            ea.profile_enable(False)
            ms = e0.elapsed_time(e1)
            gbps = p["expand_bytes"] / (p["expand_ms"] / 1e3) / 1e9
            rec = {"config": name, "labels": labels, "n": g.n, "step_ms": ms, "entries_per_s": g.n * g.n / (ms / 1e3),
                   "expand_ms": p["expand_ms"], "expand_GBps": gbps, "expand_frac_of_copy_bw": gbps / peaks["hbm_gbs"],
                   "fw_ms": p["fw_phase3_ms"] + p["fw_phase2_ms"] + p["fw_phase1_ms"]}
            print(json.dumps(rec), flush=True)
            lines.append(rec)
            del out
            torch.cuda.empty_cache()
    if args.out:
        with open(args.out, "w") as f:
            for r in lines:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
