mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_partitioned.py -x -q > gpurun_out/t_part.txt 2>&1
timeout 300 python tools/part_scan.py --parts 1,2,4,8 --apps bfs --reps 2 > gpurun_out/rt_bfs.txt 2>&1
: > gpurun_out/rt_pr.txt
for cfg in "0 0.25" "1e-3 0.25" "1e-2 0.25" "1e-4 0.25" "1e-3 0.1" "1e-2 0.5"; do
  set -- $cfg
  echo "== eps0 $1 f $2" >> gpurun_out/rt_pr.txt
  ATOS_PR_EPS0=$1 ATOS_PR_EPSF=$2 timeout 300 python tools/part_scan.py --scale 23 --parts 1,2,8 --apps pr --reps 0 >> gpurun_out/rt_pr.txt 2>&1
done
