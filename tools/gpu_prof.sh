# Round profile set on cfg4: bench line, ncu launch list of one step, ncu --set full of the top kernels.
# launch picks (k_fw_tiles, the BCC root piece's FW comes first): launch 0 = round 0's phase 2, then per
# round k: cross tiles (main), round k+1's phase 2 (side), rest of round k (main) -> launch 3k+3 is the
# rest-of-round phase 3 of round k; -s 99 = round 32.  k_expand_pairs launch 0 = the caller expansion.
TAG=${1:-r02}
set -x
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.log; tail -2 gpurun_out/bench_$TAG.log
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 8000 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt --no-seeds > /dev/null 2> gpurun_out/ncu_launch_$TAG.log; tail -1 gpurun_out/ncu_launch_$TAG.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fw_tiles -s 99 -c 1 -o gpurun_out/prof_fw16_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt --no-seeds > /dev/null 2> gpurun_out/ncu_fw_$TAG.log; tail -1 gpurun_out/ncu_fw_$TAG.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fw_tiles -s 99 -c 1 -o gpurun_out/prof_fw32_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt --no-seeds --fw32 --phase2 fw > /dev/null 2> gpurun_out/ncu_fw32_$TAG.log; tail -1 gpurun_out/ncu_fw32_$TAG.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_expand_pairs -s 0 -c 1 -o gpurun_out/prof_expand_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-alt --no-seeds > /dev/null 2> gpurun_out/ncu_ex_$TAG.log; tail -1 gpurun_out/ncu_ex_$TAG.log
ls -la gpurun_out | tail -8
