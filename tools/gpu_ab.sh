# A/B of in-tree library variants on one box: bash tools/gpu_ab.sh A C ...  (libearapsp_X.so; "cur" = libearapsp.so)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for rep in 1 2; do
  for v in "$@"; do
    if [ "$v" = cur ]; then L=; else L=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_$v.so; fi
    EAR_LIB=$L timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-alt --no-cpu-baseline --no-seeds > gpurun_out/ab_$v.json 2>/dev/null
    python -c "
import json; d=json.load(open('gpurun_out/ab_$v.json')); p=d['phases_ms']; print('$v', round(d['ms_per_step'],3), 'expand', round(p['expand'],3), 'part', round(p['part'],3), 'mp', round(p['part_mp'],3), 'dec', round(p['decompose'],3))"
  done
done
