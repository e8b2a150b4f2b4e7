set -x
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv
timeout 900 python bench.py > gpurun_out/bench_r01a.json 2> gpurun_out/bench_r01a.log; tail -3 gpurun_out/bench_r01a.log; cat gpurun_out/bench_r01a.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 1200 --csv --log-file gpurun_out/launches_r01a.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2> gpurun_out/ncu_launch.log; tail -2 gpurun_out/ncu_launch.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fw_tiles -s 20 -c 2 -o gpurun_out/prof_fw_r01a python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2> gpurun_out/ncu_fw.log; tail -2 gpurun_out/ncu_fw.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_expand -c 1 -o gpurun_out/prof_expand_r01a python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2> gpurun_out/ncu_ex.log; tail -2 gpurun_out/ncu_ex.log
ls -la gpurun_out
