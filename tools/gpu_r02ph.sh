cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02ph}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_pairs -c 1 -o gpurun_out/${T}_expand python tools/one_step.py cfg4 part 1 > gpurun_out/${T}_ncu.log 2>&1; echo "ncu rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_region_final -c 1 -o gpurun_out/${T}_final python tools/one_step.py cfg4 part 1 > gpurun_out/${T}_ncu2.log 2>&1; echo "ncu2 rc=$?"
