"""Time Phase II by pieces (apsp_reduced with EAR_FLAG_BCC) on a config: one warm-up call, one timed
call (device events); prints the block structure after the solve.  EAR_NO_REREDUCE=1 disables the
re-reduction of big pieces (A/B)."""
import json, os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_duttackb17_b200 as ea
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
g = gg.config(cfg)
src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
plan = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_BCC)
D = ea.alloc_D(plan)
ea.apsp_reduced(plan, D)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
ea.apsp_reduced(plan, D)
e1.record()
torch.cuda.synchronize()
cs = int((D[::97, ::89].to(torch.int64) * 7 + 1).sum().item())
print(json.dumps({"cfg": cfg, "no_rereduce": os.environ.get("EAR_NO_REREDUCE", "0"), "phase2_ms": e0.elapsed_time(e1),
                  "bcc": plan.bcc_info(), "checksum": cs}))
