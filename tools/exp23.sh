mkdir -p gpurun_out
: > gpurun_out/b128.txt
ATOS_LIB=$PWD/variants/libatos_b128.so timeout 200 python tools/sweep.py bfs-mesh --reps 3 --grid "128:128:1,128:64:1,128:32:1,256:256:1" >> gpurun_out/b128.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_b128.so timeout 200 python tools/sweep.py bfs-road --reps 3 --grid "128:128:1,128:64:1,256:256:1" >> gpurun_out/b128.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_b128.so timeout 200 python tools/sweep.py bfs-rmat --reps 3 --grid "128:128:1,256:256:1" >> gpurun_out/b128.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_b128.so timeout 200 python tools/sweep.py pr --reps 3 --grid "128:128:1" >> gpurun_out/b128.txt 2>&1
