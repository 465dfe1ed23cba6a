set -x
D=gpurun_out/r2t4
mkdir -p $D
timeout 1500 python -m pytest tests -m "gpu and not slow" -q -x > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
timeout 900 python tools/ab.py run --tags base --apps bfs-rmat --reps 8 --rounds 2 > $D/ab.txt 2>&1
timeout 900 python tools/ab.py run --tags base --apps bfs-mesh,bfs-road,pr,gc --reps 3 --rounds 1 >> $D/ab.txt 2>&1
tail -3 $D/pytest_quick.log
