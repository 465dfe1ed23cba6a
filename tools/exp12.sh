mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_partitioned.py -x -q > gpurun_out/t_part.txt 2>&1
ATOS_ROUND_TRACE=1 timeout 300 python tools/part_scan.py --parts 1,2,4,8 --apps bfs --reps 2 > gpurun_out/rt_bfs.txt 2>&1
