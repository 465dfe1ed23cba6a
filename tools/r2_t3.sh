set -x
D=gpurun_out/r2t3
mkdir -p $D
timeout 900 python -m pytest tests/test_gpu_multiproc.py tests/test_gpu_partitioned.py tests/test_gpu_timeline.py -q -x > $D/pytest_mp.log 2>&1; echo "rc=$?" >> $D/pytest_mp.log
timeout 1200 python tools/gc_order_study.py > $D/gc_order_study.txt 2>&1
tail -2 $D/pytest_mp.log
