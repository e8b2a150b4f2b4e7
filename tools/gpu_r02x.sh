cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02x}
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -n 1
timeout 1500 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.log; echo "bench rc=$?"
python - <<'PY'
import json,os
T=os.environ.get('TAG','r02x')
l=json.loads(open(f'gpurun_out/{T}_bench.json').read().strip().splitlines()[-1])
print({k:l[k] for k in ['value','ms_per_step','gpu_launches']}, l['e2e']['value'] if l.get('e2e') else None)
print('roofline', {k:l['roofline'].get(k) for k in ['kernel','achieved','peak','frac','avg_launch_ms']})
print('expand', {k:l['roofline_expand'].get(k) for k in ['achieved','frac','avg_launch_ms']})
print('phases', {k:round(v,2) for k,v in l['phases_ms'].items() if v})
print('alt', l.get('phase2_alternatives')); print('clocks', l['clocks']); print('seeds', l.get('seeds'))
PY
