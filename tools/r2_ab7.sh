set -x
D=gpurun_out/r2ab7
mkdir -p $D
timeout 900 python tools/ab.py run --tags base,gcsp1,gcsp4,gcsp8 --apps gc --reps 3 --rounds 2 > $D/ab_gc.txt 2>&1
timeout 900 python tools/ab.py run --tags base,cred,crel,credrel --apps bfs-rmat --reps 8 --rounds 2 > $D/ab_bfs.txt 2>&1
timeout 900 python tools/ab.py run --tags base,cred,crel,credrel --apps bfs-mesh,pr --reps 3 --rounds 1 >> $D/ab_bfs.txt 2>&1
