set -x
D=gpurun_out/r2ab6
mkdir -p $D
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 > $D/gc_counts.txt 2>&1
timeout 900 python tools/ab.py run --tags base,gcsp1,gcsp4,gcsp8 --apps gc --reps 3 --rounds 2 --grid 1024:128:1,32:8:1 > $D/ab_gc.txt 2>&1
