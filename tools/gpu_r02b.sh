# round-2 check: race test red on the round-1 library / green on the new one, full GPU suite, quick bench
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
EAR_LIB=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_r01race.so timeout 600 python -m pytest tests/test_concurrency_gpu.py -q -p no:cacheprovider > gpurun_out/r02b_race_r01lib.txt 2>&1
echo "race r01 lib rc=$?"; tail -5 gpurun_out/r02b_race_r01lib.txt
timeout 600 python -m pytest tests/test_concurrency_gpu.py -q -p no:cacheprovider > gpurun_out/r02b_race_new.txt 2>&1
echo "race new lib rc=$?"; tail -3 gpurun_out/r02b_race_new.txt
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider -x --timeout 900 > gpurun_out/r02b_gpu_tests.txt 2>&1
echo "gpu tests rc=$?"; tail -15 gpurun_out/r02b_gpu_tests.txt
timeout 600 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-alt > gpurun_out/r02b_bench.json 2> gpurun_out/r02b_bench.log
echo "bench rc=$?"; cat gpurun_out/r02b_bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline_expand']['frac'], d['phases_ms'])"
