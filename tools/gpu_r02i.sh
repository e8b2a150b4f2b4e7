cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 900 > gpurun_out/r02i_gpu_tests.txt 2>&1; echo "gpu tests rc=$?"; tail -5 gpurun_out/r02i_gpu_tests.txt
timeout 1200 python bench.py --no-cpu-baseline > gpurun_out/r02i_bench.json 2> gpurun_out/r02i_bench.log; echo "bench rc=$?"; tail -2 gpurun_out/r02i_bench.log
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r02i_bench.json").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"], d["roofline"]["frac"], d["roofline_expand"], d["phases_ms"], d["e2e"]["value"], d["seeds"])
PY
