cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
EAR_SSSP_STATS=1 timeout 600 python tools/time_sssp.py cfg2 cfg3_f60 cfg4 --reps 1 --no-full --no-fw 2>&1 | grep -E "^\[sssp16" | sort -u
timeout 900 python tools/time_sssp.py cfg1 cfg2 cfg3_f60 cfg4 --reps 3 --out gpurun_out/r02t_sssp_time.jsonl 2>&1 | tail -n 4
bash tools/prof_sssp16.sh b cfg4
