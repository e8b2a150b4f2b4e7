# round-2: full N x N certification (cfg4, cfg5), int32 FW rank timing on cfg5, packed on cfg4, cfg5 row blocks
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
rm -f gpurun_out/r02c_full_verify.jsonl
EAR_VERIFY_CFG5=1 EAR_VERIFY_OUT=gpurun_out/r02c_full_verify.jsonl timeout 1500 python -m pytest tests/test_full_verify_gpu.py -q -s -p no:cacheprovider > gpurun_out/r02c_full_verify.txt 2>&1
echo "full verify rc=$?"; tail -4 gpurun_out/r02c_full_verify.txt; cat gpurun_out/r02c_full_verify.jsonl
timeout 900 python tools/rank_timing.py cfg5 --fw32 --out gpurun_out/r02c_rank_timing_cfg5_int32.jsonl > /dev/null 2> gpurun_out/r02c_rank_timing_cfg5.log
echo "rank timing cfg5 rc=$?"; cat gpurun_out/r02c_rank_timing_cfg5_int32.jsonl
timeout 600 python tools/rank_timing.py cfg4 --out gpurun_out/r02c_rank_timing_cfg4_packed.jsonl > /dev/null 2> gpurun_out/r02c_rank_timing_cfg4.log
echo "rank timing cfg4 rc=$?"; cat gpurun_out/r02c_rank_timing_cfg4_packed.jsonl
timeout 900 python tools/run_cfg5.py --phase2 bcc > gpurun_out/r02c_cfg5_bcc.json 2> gpurun_out/r02c_cfg5_bcc.log
echo "cfg5 bcc rc=$?"; cat gpurun_out/r02c_cfg5_bcc.json
