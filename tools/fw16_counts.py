"""Phase II of a config with the profile counters of the packed FW (used / fallbacks / prechecked)."""
import json, os, sys, time
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_duttackb17_b200 as ea
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg5"
flags = ea.FLAG_BCC if (len(sys.argv) < 3 or sys.argv[2] == "bcc") else 0
g = gg.config(cfg)
src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
plan = ea.ear_decompose(g.n, src, dst, w, flags=flags)
D = ea.alloc_D(plan)
ea.profile_reset(); ea.profile_enable(True)
t = time.perf_counter(); ea.apsp_reduced(plan, D); torch.cuda.synchronize(); t = time.perf_counter() - t
p = ea.profile_read()
print(json.dumps({"cfg": cfg, "flags": flags, "s": t, "fw16_used": p["fw16_used"], "fw16_fallbacks": p["fw16_fallbacks"],
                  "fw16_prechecked": p["fw16_prechecked"], "p3_16_ms": p["fw_phase3_16_ms"], "p3_ms": p["fw_phase3_ms"],
                  "rereduce_ms": p["rereduce_ms"], "bcc": plan.bcc_info() if flags else None}))
