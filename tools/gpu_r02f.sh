cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_mcb_gpu.py -q -x -p no:cacheprovider > gpurun_out/r02f_mcb_tests.txt 2>&1; echo "mcb tests rc=$?"; tail -25 gpurun_out/r02f_mcb_tests.txt
timeout 600 python tools/time_mcb.py cfg1 cfg2 --out gpurun_out/r02f_mcb_time.jsonl 2>&1 | tail -5
