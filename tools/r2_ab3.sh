set -x
D=gpurun_out/r2ab3
mkdir -p $D
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 > $D/gc_counts.txt 2>&1
timeout 900 python tools/ab.py run --tags base,gcnodefer --apps gc --reps 3 --rounds 2 > $D/ab_gc.txt 2>&1
timeout 900 python -m pytest tests -m "gpu and not slow" -q -x > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
timeout 900 python tools/ab.py run --tags base --apps bfs-rmat --reps 8 --rounds 1 > $D/ab_bfs.txt 2>&1
timeout 900 python tools/ab.py run --tags base --apps bfs-mesh,bfs-road,pr --reps 3 --rounds 1 >> $D/ab_bfs.txt 2>&1
tail -2 $D/pytest_quick.log
