cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -p no:cacheprovider -k "query" > gpurun_out/r02g_query_tests.txt 2>&1; echo "query tests rc=$?"; tail -3 gpurun_out/r02g_query_tests.txt
timeout 600 python tools/time_query.py cfg4 --out gpurun_out/r02g_query.jsonl 2> gpurun_out/r02g_query.err | cut -c1-600; tail -2 gpurun_out/r02g_query.err
timeout 900 python tools/stress_relabel.py cfg2 cfg4 --out gpurun_out/r02g_relabel.jsonl 2> gpurun_out/r02g_relabel.err; tail -2 gpurun_out/r02g_relabel.err
