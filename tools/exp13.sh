mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_partitioned.py tests/test_gpu_pagerank.py -x -q > gpurun_out/t_part.txt 2>&1
ATOS_ROUND_TRACE=1 timeout 300 python tools/part_scan.py --parts 1,2,4,8 --apps bfs --reps 2 > gpurun_out/rt_bfs.txt 2>&1
ATOS_ROUND_TRACE=1 timeout 600 python tools/part_scan.py --scale 23 --parts 1,2,8 --apps pr --reps 0 > gpurun_out/rt_pr.txt 2>&1
