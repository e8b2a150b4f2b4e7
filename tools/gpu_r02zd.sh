cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02zd}
timeout 1500 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/one_step.py cfg4 bcc_sssp 1 > /dev/null 2>&1; echo "ncu rc=$?"
python tools/launch_summary.py gpurun_out/${T}_launches.csv "one apsp_full call, cfg4, blocks + SSSP (bench route)" > gpurun_out/${T}_launches.txt 2>&1
timeout 900 python tools/time_sssp.py cfg1 cfg2 cfg3_f0 cfg3_f20 cfg3_f40 cfg3_f60 cfg3_f80 cfg4 --reps 3 --no-fw --out gpurun_out/${T}_routes.jsonl > /dev/null 2>&1; echo "routes rc=$?"
