# L2 bulk prefetch knob (EAR_XP_PF) on the expansion: correctness with 3, cfg4 A/B, cfg5 A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
EAR_XP_PF=3 timeout 600 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/pf_tests.txt 2>&1; echo "tests rc=$?"; tail -n 1 gpurun_out/pf_tests.txt
bash tools/gpu_envab.sh EAR_XP_PF "0 1 2 3"
for v in 0 3; do EAR_XP_PF=$v timeout 600 python bench.py --config cfg5 --no-e2e --no-alt --no-cpu-baseline --no-seeds --steps 3 --warmup 3 > gpurun_out/pf5.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/pf5.json')); p=d['phases_ms']; print('cfg5 PF=$v', round(d['ms_per_step'],3), 'expand', round(p['expand'],3))"; done
