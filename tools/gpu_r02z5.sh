# final-code check: smoke, the whole GPU suite, the bench line (cfg4, default), the ncu launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02z5}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/${T}_smoke.txt
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${T}_gpu_tests.txt 2>&1; echo "tests rc=$?"; tail -n 2 gpurun_out/${T}_gpu_tests.txt
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); p=d['phases_ms']; print(d['value'], d['ms_per_step'], round(p['expand'],3), d['roofline']['frac'], d['roofline_phase2']['frac'], d['e2e']['value'], d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/one_step.py cfg4 part 2 > gpurun_out/${T}_ncu_list.log 2>&1; echo "ncu list rc=$?"
python tools/launch_summary.py gpurun_out/${T}_launches.csv "cfg4, --phase2 part (bench route), 2 apsp_full steps" > gpurun_out/${T}_launches.txt; head -12 gpurun_out/${T}_launches.txt
timeout 900 python bench.py --config cfg5 --no-e2e --steps 5 --warmup 3 > gpurun_out/${T}_bench_cfg5.json 2> gpurun_out/${T}_bench_cfg5.log; echo "cfg5 bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench_cfg5.json')); p=d['phases_ms']; print(d['value'], d['ms_per_step'], round(p['expand'],3), d['roofline']['frac'], d['clocks'])"
for cfg in cfg4 cfg2; do for lab in morton random; do timeout 600 python tools/time_expand.py $cfg --labels $lab --out gpurun_out/${T}_expand_labels.jsonl > /dev/null 2>&1; echo "expand $cfg $lab rc=$?"; done; done
