cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pg}
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-alt > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); print(d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['kernel'], d['roofline']['frac'], d.get('roofline_phase2',{}).get('frac'))"
timeout 2400 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/${T}_gpu_tests.txt 2>&1; echo "tests rc=$?"; tail -n 5 gpurun_out/${T}_gpu_tests.txt
