cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python tools/one_step.py cfg4 bcc_sssp 4
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02za_launches.csv python tools/one_step.py cfg4 bcc_sssp 2 > /dev/null 2>&1; echo "ncu rc=$?"
python tools/launch_summary.py gpurun_out/r02za_launches.csv "two apsp_full calls, cfg4, blocks + SSSP" | head -40
