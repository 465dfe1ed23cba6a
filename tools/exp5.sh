mkdir -p gpurun_out
export ATOS_ROUND_TRACE=1
timeout 300 python tools/part_scan.py --parts 1,2,4 --apps bfs --reps 0 > gpurun_out/rt_bfs.txt 2>&1
timeout 300 python tools/part_scan.py --scale 23 --parts 1,2 --apps pr --reps 0 > gpurun_out/rt_pr.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_phase.so ATOS_PHASE=1 timeout 300 python tools/part_scan.py --parts 2 --apps bfs --reps 0 > gpurun_out/rt_bfs_phase.txt 2>&1
