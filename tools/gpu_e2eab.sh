# e2e A/B (apsp_full_host_async pipeline) between the in-tree library and libearapsp_prev.so, alternating
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for rep in 1 2 3; do for v in prev cur; do if [ $v = cur ]; then L=; else L=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_$v.so; fi
EAR_LIB=$L timeout 600 python bench.py --steps 3 --warmup 3 --no-alt --no-cpu-baseline --no-seeds > gpurun_out/sl.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/sl.json')); print('$v', round(d['ms_per_step'],3), 'e2e', d['e2e']['value'])"; done; done
