set -x
D=gpurun_out/r2t2
mkdir -p $D
timeout 1200 python -m pytest tests -m "gpu and not slow" -q -x > $D/pytest_quick.log 2>&1; echo "rc=$?" >> $D/pytest_quick.log
for a in bfs pr gc; do timeout 300 python tools/normalized_tp.py $a > $D/ntp_$a.txt 2>&1; done
timeout 300 python tools/normalized_tp.py bfs --mesh 4900 > $D/ntp_bfs_mesh.txt 2>&1
timeout 900 python bench.py --no-apps --no-bsp --no-cpu > $D/bench.json 2> $D/bench.err
tail -2 $D/pytest_quick.log
