cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02ze}
EAR_VERIFY_CFG5=1 EAR_VERIFY_OUT=gpurun_out/${T}_full_verify.jsonl timeout 1800 python -m pytest tests/test_full_verify_gpu.py -q -x -p no:cacheprovider -s > gpurun_out/${T}_full_verify.txt 2>&1; echo "verify rc=$?"; tail -n 2 gpurun_out/${T}_full_verify.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_sssp16 -c 1 -o gpurun_out/${T}_sssp16_bench python tools/one_step.py cfg4 bcc_sssp 1 > gpurun_out/${T}_ncu.log 2>&1; echo "ncu rc=$?"
ncu -i gpurun_out/${T}_sssp16_bench.ncu-rep --page source --csv --print-source sass > gpurun_out/${T}_sssp16_bench.sass.csv 2>&1
