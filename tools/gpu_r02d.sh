cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/expand_lab2.py cfg4 > gpurun_out/r02d_lab2.jsonl 2> gpurun_out/r02d_lab2.err
echo "lab rc=$?"; cat gpurun_out/r02d_lab2.jsonl; tail -3 gpurun_out/r02d_lab2.err
