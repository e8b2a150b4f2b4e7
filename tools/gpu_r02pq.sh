cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02pq}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/${T}_smoke.txt
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); p=d['phases_ms']; print(d['value'], d['ms_per_step'], p['expand'], p['part'], p['part_mp'], d['roofline']['frac'], d['e2e']['value'], d['seeds'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/one_step.py cfg4 part 2 > gpurun_out/${T}_ncu_list.log 2>&1; echo "ncu list rc=$?"
python tools/launch_summary.py gpurun_out/${T}_launches.csv "cfg4, --phase2 part (bench route), 2 apsp_full steps" > gpurun_out/${T}_launches.txt; head -14 gpurun_out/${T}_launches.txt
EAR_VERIFY_CFG5=1 EAR_VERIFY_OUT=gpurun_out/${T}_full_verify.jsonl timeout 1800 python -m pytest tests/test_full_verify_gpu.py -q -x -p no:cacheprovider -s -k part > gpurun_out/${T}_full_verify.txt 2>&1; echo "verify rc=$?"; tail -n 1 gpurun_out/${T}_full_verify.txt; cat gpurun_out/${T}_full_verify.jsonl | cut -c1-200
