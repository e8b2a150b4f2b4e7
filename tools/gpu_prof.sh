# Round profile set on cfg4: bench line, ncu launch list of one step, ncu --set full of the top kernels.
# launch picks: k_fw_tiles16 launch 99 = round 32 rest-of-round phase 3 (launch order per round: cross, next pivot row, rest); k_expand launch 2 = the caller expansion (0-1: the re-reduced piece expansions; --no-alt skips the untimed BCC-info solve)
TAG=${1:-r01}
set -x
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.log; tail -2 gpurun_out/bench_$TAG.log; cat gpurun_out/bench_$TAG.json
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 8000 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt > /dev/null 2> gpurun_out/ncu_launch_$TAG.log; tail -1 gpurun_out/ncu_launch_$TAG.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fw_tiles16 -s 99 -c 1 -o gpurun_out/prof_fw16_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt > /dev/null 2> gpurun_out/ncu_fw_$TAG.log; tail -1 gpurun_out/ncu_fw_$TAG.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_expand -s 2 -c 1 -o gpurun_out/prof_expand_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt > /dev/null 2> gpurun_out/ncu_ex_$TAG.log; tail -1 gpurun_out/ncu_ex_$TAG.log
ls -la gpurun_out
