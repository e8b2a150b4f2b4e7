# expansion: one row pointer per partner gather run (r_of_g) vs the previous commit's kernel (libearapsp_prev.so)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/lc2_tests.txt 2>&1; echo "tests rc=$?"; tail -n 1 gpurun_out/lc2_tests.txt
bash tools/gpu_ab.sh prev cur
