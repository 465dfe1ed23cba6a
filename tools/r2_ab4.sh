set -x
D=gpurun_out/r2ab4
mkdir -p $D
ATOS_LIB=variants/libatos_gccnt.so timeout 300 python tools/gc_counts.py 20 64 > $D/gc_counts.txt 2>&1
timeout 900 python tools/ab.py run --tags base,gcnodefer --apps gc --reps 3 --rounds 2 > $D/ab_gc.txt 2>&1
ATOS_PHASE=1 ATOS_LIB=variants/libatos_phase.so timeout 300 python tools/run_app.py bfs scale=26 reps=3 > $D/phase_bfs.txt 2>&1
ATOS_PHASE=1 ATOS_LIB=variants/libatos_phase.so timeout 300 python tools/run_app.py pr scale=22 reps=2 > $D/phase_pr.txt 2>&1
