# ncu --set full of one k_sssp16 launch (reduced APSP by SSSP on a config), with the SASS and CUDA source
# pages (stall sampling, instructions per line)
TAG=${1:-x}
CFG=${2:-cfg2}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_sssp16 -s ${SKIP:-1} -c 1 -o gpurun_out/sssp16_$TAG python tools/time_sssp.py $CFG --reps 1 --no-full --no-fw > gpurun_out/sssp16_$TAG.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/sssp16_$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/sssp16_$TAG.sass.csv 2>&1
ncu -i gpurun_out/sssp16_$TAG.ncu-rep --page source --csv --print-source cuda > gpurun_out/sssp16_$TAG.cuda.csv 2>&1
ncu -i gpurun_out/sssp16_$TAG.ncu-rep --page raw --csv > gpurun_out/sssp16_$TAG.raw.csv 2>&1
ncu -i gpurun_out/sssp16_$TAG.ncu-rep --page details --csv > gpurun_out/sssp16_$TAG.details.csv 2>&1
ls -la gpurun_out | grep sssp16_$TAG
