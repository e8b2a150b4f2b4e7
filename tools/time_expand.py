"""Time expand_ears on a config (device events, 5 repetitions after 2 warm-ups)."""
import os, sys, time, torch
sys.path.insert(0,'.')
import paper_conf_ipps_duttackb17_b200 as ea
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
g=gg.config('cfg4')
src,dst,w=(torch.as_tensor(x).cuda() for x in (g.src,g.dst,g.w))
plan=ea.ear_decompose(g.n,src,dst,w); D=ea.alloc_D(plan); ea.apsp_reduced(plan,D)
out=torch.empty((g.n,g.n),dtype=torch.int32,device='cuda')
for i in range(2): ea.expand_ears(plan,D,0,g.n,out=out)
torch.cuda.synchronize()
e0,e1=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
e0.record()
for i in range(5): ea.expand_ears(plan,D,0,g.n,out=out)
e1.record(); torch.cuda.synchronize()
print('DBG', os.environ.get('EAR_EXPAND_DEBUG','0'), 'ms', e0.elapsed_time(e1)/5)
