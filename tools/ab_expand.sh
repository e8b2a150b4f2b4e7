# A/B of expand_ears on cfg4: the previous in-tree build (libearapsp_prev.so) vs the current one
for i in 1 2; do
  EAR_LIB=$PWD/paper_conf_ipps_duttackb17_b200/libearapsp_prev.so timeout 300 python tools/time_expand.py | sed 's/^/prev /'
  timeout 300 python tools/time_expand.py | sed 's/^/new  /'
done
