cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02w}
timeout 900 python -m pytest tests/test_bcc_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_bcc_tests.txt 2>&1; echo "bcc tests rc=$?"; tail -n 2 gpurun_out/${T}_bcc_tests.txt
timeout 900 python -m pytest tests/test_sssp16_gpu.py tests/test_parity_gpu.py -k "sssp" -q -x -p no:cacheprovider > gpurun_out/${T}_sssp_tests.txt 2>&1; echo "sssp tests rc=$?"; tail -n 1 gpurun_out/${T}_sssp_tests.txt
timeout 900 python tools/time_sssp.py cfg2 cfg3_f60 cfg4 --reps 3 --no-fw --out gpurun_out/${T}_sssp_time.jsonl 2>&1 | tail -n 3
