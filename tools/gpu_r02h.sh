cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
rm -f gpurun_out/r02h_expand_ab.jsonl
timeout 900 python tools/time_expand.py cfg4 --out gpurun_out/r02h_expand_ab.jsonl 2>&1 | tail -3
timeout 900 python tools/time_expand.py cfg4 --labels random --out gpurun_out/r02h_expand_ab.jsonl 2>&1 | tail -3
timeout 900 python tools/time_expand.py cfg2 --out gpurun_out/r02h_expand_ab.jsonl 2>&1 | tail -3
timeout 900 python tools/time_expand.py cfg2 --labels random --out gpurun_out/r02h_expand_ab.jsonl 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 900 > gpurun_out/r02h_gpu_tests.txt 2>&1; echo "gpu tests rc=$?"; tail -15 gpurun_out/r02h_gpu_tests.txt
