cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02zc}
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/${T}_gpu_tests.txt 2>&1; echo "gpu tests rc=$?"; tail -n 3 gpurun_out/${T}_gpu_tests.txt
EAR_SSSP_STATS=1 timeout 1200 python tools/time_sssp.py cfg5 --reps 1 --no-full --no-fw --out gpurun_out/${T}_cfg5.jsonl 2>&1 | grep -E "^\[sssp|config" | sort -u | head
