# lab: expansion with the partner gathers (EAR_XP_PF=4) / all gathers (12) cut (wrong output, timing only)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
EAR_XP_PIPE=0 bash tools/gpu_envab.sh EAR_XP_PF "0 4 12 1 5"
