set -x
D=gpurun_out/r2ab2
mkdir -p $D
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 > $D/gc_counts.txt 2>&1
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 worker=32 fetch_size=8 >> $D/gc_counts.txt 2>&1
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 conflict_policy=2 >> $D/gc_counts.txt 2>&1
timeout 900 python tools/ab.py run --tags base,pf,bo256,bo256pf --apps bfs-mesh,bfs-road --reps 3 --rounds 2 > $D/ab_mesh.txt 2>&1
