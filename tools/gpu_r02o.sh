cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_sssp16_gpu.py -q -x -p no:cacheprovider > gpurun_out/r02o_sssp16_tests.txt 2>&1; echo "sssp16 tests rc=$?"; tail -5 gpurun_out/r02o_sssp16_tests.txt
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -p no:cacheprovider -k "sssp" > gpurun_out/r02o_sssp_parity.txt 2>&1; echo "sssp parity rc=$?"; tail -3 gpurun_out/r02o_sssp_parity.txt
EAR_SSSP_STATS=1 timeout 900 python tools/time_sssp.py cfg1 cfg2 --reps 1 --no-full --no-fw 2>&1 | grep -E "sssp16|config" | head
timeout 1200 python tools/time_sssp.py cfg1 cfg2 cfg3_f60 cfg4 --out gpurun_out/r02o_sssp_time.jsonl 2>&1 | tail -6
EAR_SSSP16_NT=512 timeout 1200 python tools/time_sssp.py cfg4 --no-fw --out gpurun_out/r02o_sssp_time_nt512.jsonl 2>&1 | tail -2
