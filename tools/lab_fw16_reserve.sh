# dynamic FW16 (variant 9): slots left free by the rest-of-round launch for the next round's pivot chain
for r in 0 4 8 16 0 4 8 16; do EAR_FW16_VARIANT=9 EAR_FW16_RESERVE=$r timeout 300 python tools/sweep_fw16.py --one cfg4 | sed "s/^/r$r /"; done
for r in 0 8; do EAR_FW16_VARIANT=9 EAR_FW16_RESERVE=$r EAR_FW16_LOOKAHEAD=0 timeout 300 python tools/sweep_fw16.py --one cfg4 | sed "s/^/nola r$r /"; done
