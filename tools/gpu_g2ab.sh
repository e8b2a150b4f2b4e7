cd $GRAFT_REPO_ROOT
for cfg in cfg4 cfg5; do for v in A G2; do
  EAR_XP_GP=1 EAR_LIB=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_$v.so timeout 600 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-alt --no-cpu-baseline --no-seeds > gpurun_out/g2.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/g2.json')); print('$cfg $v', round(d['ms_per_step'],3), 'expand', round(d['phases_ms']['expand'],3))"
done; done
