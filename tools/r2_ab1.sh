set -x
D=gpurun_out/r2ab1
mkdir -p $D
timeout 900 python -m pytest tests -m "gpu and not slow" -q -x > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
timeout 900 python tools/ab.py run --tags base,lbs,pf --apps bfs-rmat --reps 8 --rounds 2 > $D/ab_bfs.txt 2>&1
timeout 600 python tools/ab.py run --tags base,lbs,pf --apps bfs-mesh,pr,bfs-road --reps 3 --rounds 1 > $D/ab_other.txt 2>&1
timeout 600 python bench.py --no-apps --no-bsp --no-cpu > $D/bench.json 2> $D/bench.err
tail -2 $D/pytest_quick.log
