# ncu capture of the lane-consecutive expansion + the partner-row L2 prefetch knob A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
T=${TAG:-r02lc}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_pairs -c 1 -o gpurun_out/${T}_expand python tools/one_step.py cfg4 part 1 > gpurun_out/${T}_ncu_e.log 2>&1; echo "ncu expand rc=$?"
bash tools/gpu_envab.sh EAR_XP_PF "0 1"
