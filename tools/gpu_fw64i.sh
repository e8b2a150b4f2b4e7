# int32 64-tile boundary FW: region-route tests, cfg5 trace and one-call timing, cfg4 bench line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02fi}
timeout 900 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_part_tests.txt 2>&1; echo "tests rc=$?"; tail -n 2 gpurun_out/${T}_part_tests.txt
EAR_PART_TRACE=1 timeout 600 python tools/one_step.py cfg5 part 2 > gpurun_out/${T}_cfg5_trace.txt 2>&1; echo "trace rc=$?"; grep -i "fw\|total\|ms" gpurun_out/${T}_cfg5_trace.txt | tail -40
timeout 900 python bench.py --config cfg5 --no-e2e --steps 5 --warmup 3 > gpurun_out/${T}_cfg5_bench.json 2> gpurun_out/${T}_cfg5_bench.log; echo "cfg5 bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_cfg5_bench.json')); print(d['value'], d['ms_per_step'], d['phases_ms'])"
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); print(d['value'], d['ms_per_step'], d['phases_ms'])"
