L=gpurun_out/rg3.log; : > $L
for mode in nolaunch graph host; do
  unset ABFT_RESTART_HOST_WAIT ABFT_DBG_RESTART_GRAPH_NOLAUNCH
  [ $mode = host ] && export ABFT_RESTART_HOST_WAIT=1
  [ $mode = nolaunch ] && export ABFT_DBG_RESTART_GRAPH_NOLAUNCH=1
  echo "== $mode" >> $L
  timeout 300 python tools/potrf_profile.py 30720 512 1 3 >> $L 2>&1
done
