cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pc}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/${T}_smoke.txt
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); print(d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['kernel'], d['roofline']['frac'], d.get('roofline_phase2',{}).get('frac'), d['e2e'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/one_step.py cfg4 part 2 > gpurun_out/${T}_ncu_list.log 2>&1; echo "ncu list rc=$?"
python tools/launch_summary.py gpurun_out/${T}_launches.csv "cfg4 part, 2 steps" > gpurun_out/${T}_launches.txt; head -30 gpurun_out/${T}_launches.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_region -c 3 -o gpurun_out/${T}_region python tools/one_step.py cfg4 part 1 > gpurun_out/${T}_ncu.log 2>&1; echo "ncu full rc=$?"
EAR_VERIFY_CFG5=1 EAR_VERIFY_OUT=gpurun_out/${T}_full_verify.jsonl timeout 1800 python -m pytest tests/test_full_verify_gpu.py -q -x -p no:cacheprovider -s -k part > gpurun_out/${T}_full_verify.txt 2>&1; echo "verify rc=$?"; tail -n 3 gpurun_out/${T}_full_verify.txt; cat gpurun_out/${T}_full_verify.jsonl
