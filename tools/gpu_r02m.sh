cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_mcb_gpu.py -q -x -p no:cacheprovider > gpurun_out/r02m_mcb_tests.txt 2>&1; echo "mcb tests rc=$?"; tail -3 gpurun_out/r02m_mcb_tests.txt
timeout 900 python tools/time_mcb.py cfg1 cfg2 --out gpurun_out/r02m_mcb_time.jsonl 2>&1 | tail -2
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r02m_mcb_launches.csv python tools/time_mcb.py cfg2 > /dev/null 2>&1; echo "ncu rc=$?"
python tools/launch_summary.py gpurun_out/r02m_mcb_launches.csv "first 600 launches of ear_mcb on cfg2 (build + ~130 phases)" | head -16
