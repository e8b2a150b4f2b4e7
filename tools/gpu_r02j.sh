cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python tools/ab_compose.py cfg4 > gpurun_out/r02j_ab_compose.jsonl 2> gpurun_out/r02j_ab.err; cat gpurun_out/r02j_ab_compose.jsonl; tail -2 gpurun_out/r02j_ab.err
