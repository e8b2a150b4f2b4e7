cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r02e_smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/r02e_smoke.log
(cd microbench && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o minplus_peak minplus_peak.cu && ./minplus_peak) > gpurun_out/r02e_minplus_peak.jsonl 2>&1; cat gpurun_out/r02e_minplus_peak.jsonl
timeout 1200 python bench.py > gpurun_out/r02e_bench.json 2> gpurun_out/r02e_bench.log; echo "bench rc=$?"; tail -3 gpurun_out/r02e_bench.log
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02e_bench.json").read().strip().splitlines()[-1])
for k in ("value", "ms_per_step", "gpu_launches", "step_ms", "seeds", "profiled_pass", "clocks", "e2e", "cpu_baseline"):
    print(k, json.dumps(d.get(k))[:600])
print("roofline", d["roofline"]["frac"], d["roofline_expand"]["frac"])
PY
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r02e_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-alt --no-seeds > /dev/null 2>&1; echo "ncu rc=$?"; wc -l gpurun_out/r02e_launches.csv
