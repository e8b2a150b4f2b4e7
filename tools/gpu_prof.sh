# ncu captures of the two dominant kernels on cfg4 (one bench step, no warm-up), plus the host timeline
TAG=${1:-r01}
python tools/host_timeline.py cfg4 2>&1 | tail -5
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fw_tiles -s 21 -c 1 -o gpurun_out/prof_fw_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2> gpurun_out/ncu_fw_$TAG.log; tail -1 gpurun_out/ncu_fw_$TAG.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_expand -c 1 -o gpurun_out/prof_expand_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2> gpurun_out/ncu_ex_$TAG.log; tail -1 gpurun_out/ncu_ex_$TAG.log
