set -x
mkdir -p gpurun_out
G="256:256:1,256:512:1,256:1024:1,512:512:1,512:1024:1,128:128:1,128:256:1,128:512:1,1024:1024:1"
timeout 300 python tools/sweep.py bfs-rmat --reps 5 --grid $G > gpurun_out/sw_bfs_def.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_ku8.so timeout 300 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1,256:512:1,128:256:1,512:512:1" > gpurun_out/sw_bfs_ku8.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_ku2.so timeout 300 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1,256:512:1,128:256:1" > gpurun_out/sw_bfs_ku2.txt 2>&1
timeout 300 python tools/sweep.py pr --reps 3 --grid "256:256:1,256:512:1,256:1024:1,512:512:1,128:256:1,128:128:1" > gpurun_out/sw_pr_def.txt 2>&1
ATOS_LIB=$PWD/variants/libatos_ku8.so timeout 300 python tools/sweep.py pr --reps 3 --grid "256:256:1,256:512:1" > gpurun_out/sw_pr_ku8.txt 2>&1
timeout 300 python tools/sweep.py bfs-mesh --reps 3 --grid "256:256:1,128:128:1,256:512:1,64:64:1" > gpurun_out/sw_mesh_def.txt 2>&1
