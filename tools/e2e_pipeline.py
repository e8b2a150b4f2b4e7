"""Host timeline of pipelined apsp_full_host_async calls on cfg4: time of each enqueue return and each
wait return (seconds from the start), and the synchronous apsp_full_host for comparison."""
import json, os, sys, time
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_duttackb17_b200 as ea
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
g = gg.config(sys.argv[1] if len(sys.argv) > 1 else "cfg4")
K = int(sys.argv[2]) if len(sys.argv) > 2 else 4
hs, hd, hw = (torch.as_tensor(x).pin_memory() for x in (g.src, g.dst, g.w))
hout = torch.empty((g.n, g.n), dtype=torch.int32, pin_memory=True)
st = torch.cuda.current_stream()
ea.apsp_full_host(g.n, hs, hd, hw, out=hout, flags=ea.FLAG_BCC, stream=st)
if "--warm2" in sys.argv:   # two jobs in flight once: the memory pool reaches its pipelined size
    for j in [ea.apsp_full_host_async(g.n, hs, hd, hw, out=hout, flags=ea.FLAG_BCC, stream=st) for _ in range(2)]:
        j.wait()
t0 = time.perf_counter()
for _ in range(2):
    ea.apsp_full_host(g.n, hs, hd, hw, out=hout, flags=ea.FLAG_BCC, stream=st)
sync_s = (time.perf_counter() - t0) / 2
ev = []
t0 = time.perf_counter()
prev = None
for i in range(K):
    j = ea.apsp_full_host_async(g.n, hs, hd, hw, out=hout, flags=ea.FLAG_BCC, stream=st)
    ev.append(("enq", i, time.perf_counter() - t0))
    if prev is not None:
        prev.wait()
        ev.append(("wait", i - 1, time.perf_counter() - t0))
    prev = j
prev.wait()
ev.append(("wait", K - 1, time.perf_counter() - t0))
print(json.dumps({"sync_s_per_call": sync_s, "timeline": ev, "pipelined_s_per_call": ev[-1][2] / K}))
