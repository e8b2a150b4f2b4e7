# split-barrier k_fw64 (EAR_FW64_SPLIT=1): correctness under a timeout first, then timing
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
EAR_FW64_SPLIT=1 timeout 400 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/split_tests.txt 2>&1; rc=$?; echo "tests rc=$rc"; tail -n 2 gpurun_out/split_tests.txt
if [ $rc -ne 0 ]; then exit 0; fi
for v in 0 1; do EAR_FW64_SPLIT=$v EAR_PART_TRACE=1 timeout 120 python tools/one_step.py cfg4 part 2 2>&1 | grep "fw64" | tail -1; done
bash tools/gpu_envab.sh EAR_FW64_SPLIT "0 1"
