set -x
D=gpurun_out/r2t5
mkdir -p $D
timeout 1500 python -m pytest tests -m "gpu and not slow" -q > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
timeout 900 python tools/ab.py run --tags base,nofuse --apps bfs-mesh,bfs-road --reps 3 --rounds 2 > $D/ab.txt 2>&1
timeout 900 python tools/ab.py run --tags base,nofuse --apps bfs-rmat --reps 8 --rounds 2 >> $D/ab.txt 2>&1
tail -3 $D/pytest_quick.log
