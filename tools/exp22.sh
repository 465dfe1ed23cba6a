# NEXT-2 / NEXT-3 study outputs (design-space sweep, colouring ordering study, progress timelines)
mkdir -p gpurun_out
timeout 400 python tools/sweep.py bfs-rmat --reps 3 --grid "1:1:1,1:4:1,32:1:1,32:4:1,32:16:1,64:64:1,128:128:1,256:64:1,256:256:1,512:512:1,1024:1024:1,256:256:0,32:8:0" > gpurun_out/study_sweep_bfs_rmat.txt 2>&1
timeout 400 python tools/sweep.py bfs-mesh --reps 2 --grid "1:4:1,32:4:1,32:8:1,64:64:1,128:128:1,256:256:1,256:256:0,32:8:0" > gpurun_out/study_sweep_bfs_mesh.txt 2>&1
timeout 400 python tools/sweep.py pr --reps 2 --grid "1:1:1,32:4:1,32:8:1,128:128:1,256:256:1,512:512:1,1024:1024:1,256:256:0,512:512:0" > gpurun_out/study_sweep_pr.txt 2>&1
timeout 400 python tools/sweep.py gc --reps 2 --grid "1:1:1,32:8:1,256:128:1,512:128:1,1024:128:1,1024:128:0,32:8:0" > gpurun_out/study_sweep_gc.txt 2>&1
timeout 400 python tools/sweep.py gc --reps 2 --grid "32:8:1,1024:128:1,1024:128:0,32:8:0" --extra permute_init=1 > gpurun_out/study_sweep_gc_permuted.txt 2>&1
TL_ROWS=30 timeout 300 python tools/run_app.py bfs scale=26 timeline=20000 > gpurun_out/study_timeline_bfs_c5.txt 2>&1
TL_ROWS=30 timeout 300 python tools/run_app.py pr scale=22 timeline=20000 > gpurun_out/study_timeline_pr_c3.txt 2>&1
TL_ROWS=30 timeout 300 python tools/run_app.py gc scale=20 ef=64 timeline=20000 > gpurun_out/study_timeline_gc_c4.txt 2>&1
