mkdir -p gpurun_out
ATOS_ROUND_TRACE=1 ATOS_LIB=$PWD/variants/libatos_skipremote.so timeout 300 python tools/part_scan.py --parts 1,2 --apps bfs --reps 1 > gpurun_out/skipremote.txt 2>&1
