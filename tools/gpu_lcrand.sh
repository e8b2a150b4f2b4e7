# staged (EAR_XP_GP=0) vs global one-CTA (2) partners under Morton and random labels, time_expand (non-CONN kernel)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for lc in 0 2; do for lab in morton random; do EAR_XP_GP=$lc timeout 600 python tools/time_expand.py cfg4 --labels $lab 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l)
  if d['kernel']=='pairs': print('GP=$lc', d['labels'], round(d['kernel_ms'],3))"; done; done
