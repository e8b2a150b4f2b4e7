cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for pm in 2048 4096; do
  echo "== EAR_PREC_MIN=$pm"
  EAR_PREC_MIN=$pm EAR_PART_TRACE=1 python tools/one_step.py cfg4 part 2 2>&1 | tail -14 | grep "fw\|H solved\|step\|n="
  EAR_PREC_MIN=$pm python tools/one_step.py cfg5 part 3 2>&1 | tail -1
done
timeout 900 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -2
EAR_PREC_MIN=100000 timeout 900 python -m pytest tests/test_part_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -2
