set -x
D=gpurun_out/r2ab8
mkdir -p $D
timeout 1200 python -m pytest tests -m "gpu and not slow" -q -x > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
timeout 900 python tools/ab.py run --tags base,nofuse --apps bfs-rmat --reps 8 --rounds 3 > $D/ab_bfs.txt 2>&1
timeout 900 python tools/ab.py run --tags base,nofuse --apps bfs-mesh,bfs-road --reps 3 --rounds 2 >> $D/ab_bfs.txt 2>&1
ATOS_TRACE=1 E2E_STEPS=10 timeout 600 python tools/e2e_breakdown.py > $D/e2e_trace.txt 2>&1
tail -2 $D/pytest_quick.log
