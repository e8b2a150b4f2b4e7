cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_mcb_gpu.py -q -x -p no:cacheprovider > gpurun_out/r02n_mcb_tests.txt 2>&1; echo "mcb tests rc=$?"; tail -3 gpurun_out/r02n_mcb_tests.txt
timeout 900 python tools/time_mcb.py cfg1 cfg2 --out gpurun_out/r02n_mcb_time.jsonl 2>&1 | tail -2
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/r02n_sanitize_$tool.txt 2>&1
  echo "sanitize $tool rc=$?"; tail -3 gpurun_out/r02n_sanitize_$tool.txt
done
