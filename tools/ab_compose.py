"""A/B of one apsp_full step on cfg4 (FLAG_BCC): the u16 route (Phase II composes D's u16 rows, the
pair-major expansion stages them) against the int32 route (EAR_EXPAND_PAIRS=0: int32 D, row-group
expansion); per-phase device times from the library profile, 3 steps each after a warm-up."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402

g = gg.config(sys.argv[1] if len(sys.argv) > 1 else "cfg4")
src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
for mode in ("u16", "int32", "u16"):
    os.environ["EAR_EXPAND_PAIRS"] = "1" if mode == "u16" else "0"
    ea.apsp_full(g.n, src, dst, w, out=out, flags=ea.FLAG_BCC)
    torch.cuda.synchronize()
    ea.profile_reset()
    ea.profile_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        ea.apsp_full(g.n, src, dst, w, out=out, flags=ea.FLAG_BCC)
    e1.record()
    torch.cuda.synchronize()
    p = ea.profile_read()
    ea.profile_enable(False)
    keys = ["decompose_ms", "bcc_prepare_ms", "rereduce_ms", "bcc_pieces_ms", "compose_ms", "fw_phase3_ms", "expand_ms",
            "expand_d16_ms", "fw16_conv_ms"]
    print(json.dumps({"route": mode, "step_ms": e0.elapsed_time(e1) / 3, **{k: p[k] / 3 for k in keys}}), flush=True)
