cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
rm -f gpurun_out/r02l_expand_ab.jsonl
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 900 > gpurun_out/r02l_gpu_tests.txt 2>&1; echo "gpu tests rc=$?"; tail -3 gpurun_out/r02l_gpu_tests.txt
timeout 900 python tools/time_expand.py cfg4 --out gpurun_out/r02l_expand_ab.jsonl 2>&1 | cut -c1-400 | tail -2
timeout 900 python tools/time_expand.py cfg4 --labels random --out gpurun_out/r02l_expand_ab.jsonl 2>&1 | cut -c1-400 | tail -2
timeout 900 python tools/time_mcb.py cfg1 cfg2 --out gpurun_out/r02l_mcb_time.jsonl 2>&1 | tail -2
