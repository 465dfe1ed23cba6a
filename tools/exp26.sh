mkdir -p gpurun_out
: > gpurun_out/defer.txt
for c in 0 0.03 0.1 0.3 1; do
  echo "== defer $c" >> gpurun_out/defer.txt
  ATOS_PR_DEFER=$c timeout 300 python tools/part_scan.py --scale 23 --parts 1,2,8 --apps pr --reps 1 >> gpurun_out/defer.txt 2>&1
done
timeout 600 python -m pytest tests/test_gpu_partitioned.py -q -x > gpurun_out/t_part.txt 2>&1
ATOS_PR_DEFER=0.1 timeout 600 python -m pytest tests/test_gpu_partitioned.py -q -x >> gpurun_out/t_part.txt 2>&1
