cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02u}
timeout 900 python -m pytest tests/test_sssp16_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_sssp16_tests.txt 2>&1; echo "sssp16 tests rc=$?"; tail -n 1 gpurun_out/${T}_sssp16_tests.txt
EAR_SSSP16_DIST=2 timeout 900 python -m pytest tests/test_sssp16_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_sssp16_tests_u16.txt 2>&1; echo "sssp16 tests (u16 rows) rc=$?"; tail -n 1 gpurun_out/${T}_sssp16_tests_u16.txt
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -p no:cacheprovider -k "sssp" > gpurun_out/${T}_sssp_parity.txt 2>&1; echo "sssp parity rc=$?"; tail -n 1 gpurun_out/${T}_sssp_parity.txt
EAR_SSSP_STATS=1 timeout 600 python tools/time_sssp.py cfg2 cfg3_f60 cfg4 --reps 1 --no-full --no-fw 2>&1 | grep -E "^\[sssp16" | sort -u
timeout 900 python tools/time_sssp.py cfg2 cfg3_f60 cfg4 --reps 3 --no-fw --out gpurun_out/${T}_sssp_time.jsonl 2>&1 | tail -n 3
bash tools/prof_sssp16.sh ${T} cfg4 | grep rc
