set -x
D=gpurun_out/r2ab5
mkdir -p $D
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 > $D/gc_counts.txt 2>&1
timeout 900 python tools/ab.py run --tags base,gcsp1,gcsp2,gcsp8 --apps gc --reps 3 --rounds 2 > $D/ab_gc.txt 2>&1
timeout 900 python -m pytest tests -m "gpu and not slow" -q -x > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
tail -2 $D/pytest_quick.log
