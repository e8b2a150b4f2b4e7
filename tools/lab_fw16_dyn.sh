# dynamic tile scheduling (variants 8, 9) vs the static default (4): parity, cfg4 plain-FW time, per-CTA residency
for v in 8 9; do EAR_FW16_VARIANT=$v timeout 600 python -m pytest tests/test_fw16_gpu.py tests/test_bcc_gpu.py -q -x 2>&1 | tail -1; done
for v in 4 8 9 4 8 9; do EAR_FW16_VARIANT=$v timeout 300 python tools/sweep_fw16.py --one cfg4 | sed "s/^/v$v /"; done
EAR_FW16_VARIANT=8 timeout 300 python tools/fw16_cta_times.py 99
EAR_FW16_VARIANT=8 timeout 600 python tools/rank_timing.py cfg4
