# locality-adaptive expansion variant: tests, label-stress timing, bench A/B against the previous commit
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_part_gpu.py tests/test_parity_gpu.py -q -x -p no:cacheprovider > gpurun_out/loc_tests.txt 2>&1; echo "tests rc=$?"; tail -n 1 gpurun_out/loc_tests.txt
for cfg in cfg4 cfg2; do for lab in morton random; do timeout 600 python tools/time_expand.py $cfg --labels $lab --out gpurun_out/loc_expand_labels.jsonl 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
  d=json.loads(l)
  print('$cfg', d['labels'], d['kernel'], round(d['kernel_ms'],3), d['outputs_identical'])"; done; done

