set -x
D=gpurun_out/r2c2
mkdir -p $D
ATOS_PHASE=1 ATOS_LIB=variants/libatos_phase.so timeout 300 python tools/run_app.py bfs mesh=4900 reps=3 > $D/phase_mesh.txt 2>&1
ATOS_PHASE=1 ATOS_LIB=variants/libatos_phase.so timeout 300 python tools/run_app.py bfs mesh=4900 keep=0.6 reps=3 > $D/phase_road.txt 2>&1
timeout 600 python tools/sweep.py bfs-mesh --reps 2 --grid 256:256:1,256:64:1,256:32:1,128:128:1,64:64:1,32:8:1 > $D/mesh_sweep.txt 2>&1
timeout 600 python tools/sweep.py bfs-mesh --reps 2 --grid 256:256:1 --extra num_blocks=296 >> $D/mesh_sweep.txt 2>&1
timeout 600 python tools/sweep.py bfs-mesh --reps 2 --grid 256:256:1 --extra num_blocks=148 >> $D/mesh_sweep.txt 2>&1
timeout 600 python tools/sweep.py bfs-mesh --reps 2 --grid 256:256:1 --extra num_blocks=444 >> $D/mesh_sweep.txt 2>&1
