# per-variant occupancy / ALU metrics of one rest-of-round k_fw_tiles16 launch (cfg4 plain FW) + timing
for v in ${VARIANTS:-4 3 6 7}; do
  EAR_FW16_VARIANT=$v timeout 600 ncu --metrics gpu__time_duration.sum,sm__warps_active.avg.per_cycle_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k_fw_tiles16 -s 99 -c 1 --csv python tools/sweep_fw16.py --one cfg4 2>/dev/null | grep -E "gpu__time|warps_active|alu_cycles|issue_active" | sed "s/^/v$v /"
done
for v in ${VARIANTS:-4 3 6 7}; do EAR_FW16_VARIANT=$v timeout 300 python tools/sweep_fw16.py --one cfg4 | sed "s/^/v$v /"; done
