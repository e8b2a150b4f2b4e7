cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pl}
EAR_PART_TRACE=1 python tools/one_step.py cfg4 part 3 2>&1 | tail -24
EAR_PART_TRACE=1 python tools/one_step.py cfg5 part 2 2>&1 | grep "d0\|step"
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-alt --no-cpu-baseline --no-seeds > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); print(d['value'], d['ms_per_step'], d['phases_ms']['expand'], d['phases_ms']['part'], d['phases_ms']['part_mp'], d['roofline']['frac'])"
timeout 900 python -m pytest tests/test_part_gpu.py tests/test_parity_gpu.py -q -x -p no:cacheprovider > gpurun_out/${T}_tests.txt 2>&1; echo "tests rc=$?"; tail -n 2 gpurun_out/${T}_tests.txt
