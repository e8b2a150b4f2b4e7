"""Time the packed 16-bit FW on a config's plain FW (no BCC) under the development knobs of fw.cu:
phase-3 min-plus rate and FW wall time, and a checksum of D (must agree across settings).

    python tools/sweep_fw16.py [cfg4] ["LOOKAHEAD,RESERVE" ...]      (one subprocess per setting)
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
    print(json.dumps({"lookahead": os.environ.get("EAR_FW16_LOOKAHEAD", "1"), "prio": os.environ.get("EAR_FW16_PRIO", "1"),
                      "reserve": os.environ.get("EAR_FW16_RESERVE", "0"), "fw_ms": e0.elapsed_time(e1),
                      "p3_ms": p["fw_phase3_16_ms"], "p3_Tminplus": p["fw_phase3_16_minplus"] / p["fw_phase3_16_ms"] / 1e9
                      if p["fw_phase3_16_ms"] else None, "p1_ms": p["fw_phase1_ms"], "p2_ms": p["fw_phase2_ms"],
                      "conv_ms": p["fw16_conv_ms"], "used": p["fw16_used"], "checksum": cs}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--one":
        one(sys.argv[2])
        sys.exit(0)
    cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
    for setting in (sys.argv[2:] or ["0,0,1", "1,0,1", "1,0,0", "1,2,1", "1,4,1"]):
        la, rs, pr = setting.split(",")
        env = dict(os.environ, EAR_FW16_LOOKAHEAD=la, EAR_FW16_RESERVE=rs, EAR_FW16_PRIO=pr)
        subprocess.run([sys.executable, __file__, "--one", cfg], env=env, timeout=600)
