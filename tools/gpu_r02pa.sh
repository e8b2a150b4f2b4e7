cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pa}
timeout 900 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_part_tests.txt 2>&1; echo "tests rc=$?"; tail -n 15 gpurun_out/${T}_part_tests.txt
timeout 600 python bench.py --phase2 part --steps 5 --warmup 3 --no-e2e > gpurun_out/${T}_bench_part.json 2> gpurun_out/${T}_bench_part.log; echo "bench rc=$?"; tail -c 3000 gpurun_out/${T}_bench_part.json; tail -5 gpurun_out/${T}_bench_part.log
