mkdir -p gpurun_out
: > gpurun_out/c1.txt
timeout 200 python tools/sweep.py bfs-rmat --scale 16 --reps 10 --grid "256:256:1,256:64:1,128:32:1,64:16:1,32:8:1,32:4:1,256:256:0,32:8:0" >> gpurun_out/c1.txt 2>&1
timeout 200 python tools/sweep.py bfs-rmat --scale 16 --reps 10 --grid "256:256:1,256:64:1,32:8:1" --extra num_blocks=148 >> gpurun_out/c1.txt 2>&1
timeout 200 python tools/sweep.py bfs-rmat --scale 16 --reps 10 --grid "256:256:1,256:64:1,32:8:1" --extra num_blocks=296 >> gpurun_out/c1.txt 2>&1
timeout 200 python tools/sweep.py bfs-rmat --scale 16 --reps 10 --grid "256:256:1,32:8:1" --extra big_threshold=-1 >> gpurun_out/c1.txt 2>&1
