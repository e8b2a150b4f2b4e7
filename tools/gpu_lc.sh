# lane-consecutive columns in the expansion (EAR_XP_LC): correctness, cfg4 A/B, cfg5 A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_part_gpu.py tests/test_full_verify_gpu.py -q -x -p no:cacheprovider > gpurun_out/lc_tests.txt 2>&1; echo "tests rc=$?"; tail -n 3 gpurun_out/lc_tests.txt
bash tools/gpu_envab.sh EAR_XP_LC "0 1"
for v in 0 1; do EAR_XP_LC=$v timeout 600 python bench.py --config cfg5 --no-e2e --no-alt --no-cpu-baseline --no-seeds --steps 3 --warmup 3 > gpurun_out/pf5.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/pf5.json')); p=d['phases_ms']; print('cfg5 LC=$v', round(d['ms_per_step'],3), 'expand', round(p['expand'],3))"; done
