# pinned slot pool for the locality counts (no cudaHostAlloc / cudaFreeHost per plan): tests, bench A/B, e2e
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_part_gpu.py tests/test_parity_gpu.py tests/test_multiprocess_gpu.py -q -x -p no:cacheprovider > gpurun_out/slot_tests.txt 2>&1; echo "tests rc=$?"; tail -n 1 gpurun_out/slot_tests.txt
bash tools/gpu_ab.sh prev cur
for v in prev cur; do if [ $v = cur ]; then L=; else L=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_$v.so; fi
EAR_LIB=$L timeout 600 python bench.py --steps 5 --warmup 3 --no-alt --no-cpu-baseline --no-seeds > gpurun_out/sl.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/sl.json')); print('$v', round(d['ms_per_step'],3), 'e2e', d['e2e']['value'])"; done
