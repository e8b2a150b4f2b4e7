# fw64 / fw64i with two tiles' loads in flight at once: tests, cfg4 A/B, cfg5 A/B, traces
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/ld_tests.txt 2>&1; echo "tests rc=$?"; tail -n 1 gpurun_out/ld_tests.txt
bash tools/gpu_ab.sh prev cur
for v in prev cur; do if [ $v = cur ]; then L=; else L=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_$v.so; fi
EAR_LIB=$L timeout 600 python bench.py --config cfg5 --no-e2e --no-alt --no-cpu-baseline --no-seeds --steps 3 --warmup 3 > gpurun_out/pf5.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/pf5.json')); p=d['phases_ms']; print('cfg5 $v', round(d['ms_per_step'],3), 'expand', round(p['expand'],3), 'part', round(p['part'],3), 'mp', round(p['part_mp'],3))"; done
EAR_PART_TRACE=1 timeout 300 python tools/one_step.py cfg4 part 2 2>&1 | grep "fw64" | tail -1
EAR_PART_TRACE=1 timeout 300 python tools/one_step.py cfg5 part 2 2>&1 | grep "fw64" | tail -2
