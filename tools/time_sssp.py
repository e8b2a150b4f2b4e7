"""Time Phase II by per-source SSSP on a config; set EAR_SSSP_STATS=1 for round / relaxation counts."""
import sys, time, torch
sys.path.insert(0,'.')
import paper_conf_ipps_duttackb17_b200 as ea
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
g=gg.config(sys.argv[1] if len(sys.argv)>1 else 'cfg4')
src,dst,w=(torch.as_tensor(x).cuda() for x in (g.src,g.dst,g.w))
p=ea.ear_decompose(g.n,src,dst,w,flags=ea.FLAG_SSSP)
D=ea.alloc_D(p)
ea.apsp_reduced(p,D); torch.cuda.synchronize()
t=time.time(); ea.apsp_reduced(p,D); torch.cuda.synchronize(); print('sssp ms', (time.time()-t)*1e3)
