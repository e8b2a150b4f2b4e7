# Phase II knobs on cfg4 / cfg5: recursion threshold (EAR_PREC_MIN) and region seed spacing (EAR_PSEED)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
bash tools/gpu_envab.sh EAR_PREC_MIN "2048 1024 600"
bash tools/gpu_envab.sh EAR_PSEED "160 120 200"
for v in 2048 1024; do EAR_PREC_MIN=$v timeout 600 python bench.py --config cfg5 --no-e2e --no-alt --no-cpu-baseline --no-seeds --steps 3 --warmup 3 > gpurun_out/pf5.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/pf5.json')); p=d['phases_ms']; print('cfg5 PREC_MIN=$v', round(d['ms_per_step'],3), 'expand', round(p['expand'],3), 'part', round(p['part'],3), 'mp', round(p['part_mp'],3))"; done
