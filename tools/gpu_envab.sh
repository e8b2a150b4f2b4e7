# A/B of an environment knob on one box: bash tools/gpu_envab.sh VAR "val1 val2 ..." ("-" = unset)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
VAR=$1
for rep in 1 2; do
  for v in $2; do
    if [ "$v" = "-" ]; then unset $VAR; else export $VAR=$v; fi
    timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-alt --no-cpu-baseline --no-seeds > gpurun_out/envab.json 2>/dev/null
    python -c "
import json; d=json.load(open('gpurun_out/envab.json')); p=d['phases_ms']; print('$VAR=$v', round(d['ms_per_step'],3), 'expand', round(p['expand'],3), 'part', round(p['part'],3), 'mp', round(p['part_mp'],3))"
  done
done
unset $VAR
