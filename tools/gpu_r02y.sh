cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02y}
timeout 900 python -m pytest tests/test_sssp16_gpu.py tests/test_parity_gpu.py -k "sssp" -q -x -p no:cacheprovider > gpurun_out/${T}_sssp_tests.txt 2>&1; echo "sssp tests rc=$?"; tail -n 3 gpurun_out/${T}_sssp_tests.txt
EAR_SSSP16_DIST=2 timeout 900 python -m pytest tests/test_sssp16_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_sssp16_u16.txt 2>&1; echo "sssp16 (u16 rows) rc=$?"; tail -n 1 gpurun_out/${T}_sssp16_u16.txt
timeout 900 python -m pytest tests/test_bcc_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_bcc_tests.txt 2>&1; echo "bcc tests rc=$?"; tail -n 1 gpurun_out/${T}_bcc_tests.txt
EAR_SSSP_STATS=1 timeout 600 python tools/time_sssp.py cfg4 --reps 1 --no-full --no-fw 2>&1 | grep -E "^\[sssp16" | sort -u
timeout 900 python tools/time_sssp.py cfg2 cfg3_f60 cfg4 --reps 3 --no-fw --out gpurun_out/${T}_sssp_time.jsonl 2>&1 | tail -n 3
EAR_SSSP_REUSE=0 timeout 900 python tools/time_sssp.py cfg4 --reps 3 --no-fw --out gpurun_out/${T}_sssp_time_noreuse.jsonl 2>&1 | tail -n 1
