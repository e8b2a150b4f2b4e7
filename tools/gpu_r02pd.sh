cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pd}
timeout 1500 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_part_tests.txt 2>&1; echo "tests rc=$?"; tail -n 5 gpurun_out/${T}_part_tests.txt
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-alt > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); print(d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['kernel'], d['roofline']['frac'], d.get('roofline_phase2',{}).get('frac'))"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/one_step.py cfg4 part 2 > gpurun_out/${T}_ncu_list.log 2>&1; echo "ncu list rc=$?"
python tools/launch_summary.py gpurun_out/${T}_launches.csv "cfg4 part, 2 steps" > gpurun_out/${T}_launches.txt; head -16 gpurun_out/${T}_launches.txt
