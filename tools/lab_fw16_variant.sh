for v in ${VARIANTS:-0 1 2 0 1 2}; do EAR_FW16_VARIANT=$v timeout 300 python tools/sweep_fw16.py --one cfg4 | sed "s/^/{\"variant\": $v, \"r\": /; s/$/}/"; done > gpurun_out/fw16_lar.jsonl 2>&1
for v in ${TESTV:-1 2}; do EAR_FW16_VARIANT=$v timeout 600 python -m pytest tests/test_fw16_gpu.py -x -q 2>&1 | tail -1; done
cat gpurun_out/fw16_lar.jsonl
