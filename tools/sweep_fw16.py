"""Sweep the packed 16-bit FW tile-kernel configurations (EAR_FW16_VARIANT) on a config's plain FW:
phase-3 min-plus rate from the library profile, and a checksum of D (must agree across variants).

    python tools/sweep_fw16.py [cfg4] [variants...]      (one subprocess per variant)
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def one(cfg):
    sys.path.insert(0, ROOT)
    import torch
    import paper_conf_ipps_duttackb17_b200 as ea
    from paper_conf_ipps_duttackb17_b200 import graphgen as gg
    g = gg.config(cfg)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w)
    D = ea.alloc_D(plan)
    ea.apsp_reduced(plan, D)   # warm-up
    torch.cuda.synchronize()
    ea.profile_reset()
    ea.profile_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ea.apsp_reduced(plan, D)
    e1.record()
    torch.cuda.synchronize()
    p = ea.profile_read()
    cs = int((D[::97, ::89].to(torch.int64) * 7 + 1).sum().item())
    print(json.dumps({"variant": int(os.environ.get("EAR_FW16_VARIANT", "0")), "fw_ms": e0.elapsed_time(e1),
                      "p3_ms": p["fw_phase3_16_ms"], "p3_Tminplus": p["fw_phase3_16_minplus"] / p["fw_phase3_16_ms"] / 1e9
                      if p["fw_phase3_16_ms"] else None, "p1_ms": p["fw_phase1_ms"], "p2_ms": p["fw_phase2_ms"],
                      "conv_ms": p["fw16_conv_ms"], "used": p["fw16_used"], "checksum": cs}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--one":
        one(sys.argv[2])
        sys.exit(0)
    cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
    for v in (sys.argv[2:] or ["0", "1", "2", "3", "4", "5", "6"]):
        env = dict(os.environ, EAR_FW16_VARIANT=v)
        subprocess.run([sys.executable, __file__, "--one", cfg], env=env, timeout=600)
