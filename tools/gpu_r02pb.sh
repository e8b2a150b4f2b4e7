cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pb}
timeout 1500 python -m pytest tests/test_part_gpu.py -q -p no:cacheprovider > gpurun_out/${T}_part_tests.txt 2>&1; echo "tests rc=$?"; tail -n 25 gpurun_out/${T}_part_tests.txt
