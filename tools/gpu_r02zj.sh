cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_sssp16_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -n 1
EAR_SSSP16_NT=128 timeout 600 python -m pytest tests/test_sssp16_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -n 1
for nt in 256 128; do
  echo "== NT $nt"
  EAR_SSSP16_NT=$nt EAR_SSSP_STATS=1 timeout 600 python tools/time_sssp.py cfg2 cfg3_f80 cfg3_f60 cfg4 --reps 1 --no-full --no-fw 2>&1 | grep -E "^\[sssp16" | sort -u | grep -v "rows=5[0-9][0-9] \|rows=[0-9][0-9] \|rows=[0-9][0-9][0-9] " 
  EAR_SSSP16_NT=$nt timeout 600 python tools/time_sssp.py cfg2 cfg3_f80 cfg3_f60 cfg4 --reps 3 --no-fw --out gpurun_out/r02zj_nt${nt}.jsonl 2>&1 | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(d['config'], 'red sssp', round(d['reduced_sssp_ms'],2), 'red bcc+sssp', round(d['reduced_bcc_sssp_ms'],2), 'full bcc+sssp', round(d['full_bcc_sssp_ms'],2))"
done
