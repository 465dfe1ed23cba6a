mkdir -p gpurun_out
export ATOS_LIB=$PWD/variants/libatos_phase.so ATOS_PHASE=1
timeout 300 python tools/sweep.py bfs-rmat --reps 1 --grid "256:256:1" > gpurun_out/ph2_bfs.txt 2>&1
timeout 300 python tools/sweep.py bfs-mesh --reps 1 --grid "256:256:1" > gpurun_out/ph2_mesh.txt 2>&1
