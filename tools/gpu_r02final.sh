# Final profile set of round 2 (TAG defaults to r02z): smoke, GPU suite, bench, launch list, ncu captures,
# full-matrix certification, route table, per-rank timing.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02z}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.txt 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/${T}_smoke.txt
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${T}_gpu_tests.txt 2>&1; echo "tests rc=$?"; tail -n 2 gpurun_out/${T}_gpu_tests.txt
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/${T}_bench.json')); p=d['phases_ms']; print(d['value'], d['ms_per_step'], p, d['roofline']['frac'], d['roofline_phase2']['frac'], d['e2e']['value'], d['seeds'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches.csv python tools/one_step.py cfg4 part 2 > gpurun_out/${T}_ncu_list.log 2>&1; echo "ncu list rc=$?"
python tools/launch_summary.py gpurun_out/${T}_launches.csv "cfg4, --phase2 part (bench route), 2 apsp_full steps" > gpurun_out/${T}_launches.txt; head -16 gpurun_out/${T}_launches.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_pairs -c 1 -o gpurun_out/${T}_expand python tools/one_step.py cfg4 part 1 > gpurun_out/${T}_ncu_e.log 2>&1; echo "ncu expand rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_region_prod --launch-skip 3 -c 1 -o gpurun_out/${T}_prod python tools/one_step.py cfg4 part 1 > gpurun_out/${T}_ncu_p.log 2>&1; echo "ncu prod rc=$?"
EAR_VERIFY_CFG5=1 EAR_VERIFY_OUT=gpurun_out/${T}_full_verify.jsonl timeout 1800 python -m pytest tests/test_full_verify_gpu.py -q -x -p no:cacheprovider -s -k part > gpurun_out/${T}_full_verify.txt 2>&1; echo "verify rc=$?"; tail -n 1 gpurun_out/${T}_full_verify.txt
timeout 1500 python tools/time_routes.py --out gpurun_out/${T}_routes.jsonl > /dev/null 2>&1; echo "routes rc=$?"
timeout 600 python tools/part_rank_timing.py cfg4 --out gpurun_out/${T}_part_rank_timing_cfg4.jsonl > /dev/null 2>&1; echo "rank timing rc=$?"
for lab in morton random; do timeout 600 python tools/time_expand.py cfg4 --labels $lab --out gpurun_out/${T}_expand_labels.jsonl > /dev/null 2>&1; echo "expand cfg4 $lab rc=$?"; done
timeout 600 python tools/time_expand.py cfg2 --labels random --out gpurun_out/${T}_expand_labels.jsonl > /dev/null 2>&1; echo "expand cfg2 random rc=$?"
