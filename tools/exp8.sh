mkdir -p gpurun_out
ATOS_ROUND_TRACE=1 ATOS_LIB=$PWD/variants/libatos_phase.so ATOS_PHASE=1 timeout 300 python tools/part_scan.py --parts 1,2 --apps bfs --reps 0 > gpurun_out/rt_bfs_phase.txt 2>&1
for cfg in "1e-2 0.85" "1e-1 0.85" "1e-2 0.7"; do
  set -- $cfg
  echo "== eps0 $1 f $2" >> gpurun_out/rt_pr2.txt
  ATOS_PR_EPS0=$1 ATOS_PR_EPSF=$2 timeout 300 python tools/part_scan.py --scale 23 --parts 2 --apps pr --reps 0 >> gpurun_out/rt_pr2.txt 2>&1
done
