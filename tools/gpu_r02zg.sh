cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for dl in 460 920 1840 3680 7360 14720; do
  echo "== delta $dl"
  EAR_SSSP_DELTA=$dl EAR_SSSP_STATS=1 timeout 600 python tools/time_sssp.py cfg4 --reps 1 --no-full --no-fw 2>&1 | grep -E "^\[sssp16.*K=8 dist=u16" | sort -u | head -1
  EAR_SSSP_DELTA=$dl timeout 600 python tools/time_sssp.py cfg4 cfg3_f40 --reps 3 --no-fw --out gpurun_out/r02zg_delta${dl}.jsonl 2>&1 | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(d['config'], 'full bcc+sssp', round(d['full_bcc_sssp_ms'],2), 'red bcc+sssp', round(d['reduced_bcc_sssp_ms'],2))"
done
