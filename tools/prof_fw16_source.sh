# ncu --set full of one k_fw_tiles16 launch on cfg4's plain FW, with SASS-level source page (stall sampling)
TAG=${1:-x}
export EAR_FW16_VARIANT=${EAR_FW16_VARIANT:-0}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fw_tiles16 -s 300 -c 1 -o gpurun_out/fw16src_$TAG python tools/sweep_fw16.py --one cfg4 > gpurun_out/fw16src_$TAG.log 2>&1
ncu -i gpurun_out/fw16src_$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/fw16src_$TAG.sass.csv 2>&1
ncu -i gpurun_out/fw16src_$TAG.ncu-rep --page raw --csv > gpurun_out/fw16src_$TAG.raw.csv 2>&1
ls -la gpurun_out | tail -5
