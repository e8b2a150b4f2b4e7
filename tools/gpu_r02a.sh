set -x
cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nproc; lscpu | grep -i "model name"; free -g
timeout 120 ./microbench/ipc_probe > gpurun_out/r02a_ipc_probe.jsonl 2>&1; echo "ipc rc=$?"
cat gpurun_out/r02a_ipc_probe.jsonl
EAR_LIB=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_r01race.so timeout 900 python -m pytest tests/test_concurrency_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/r02a_race_old.txt
cat gpurun_out/r02a_race_old.txt
