mkdir -p gpurun_out
: > gpurun_out/requeue.txt
for cfg in "0 32" "0.1 32" "1 32" "10 32" "100 32" "10 256" "100 1024"; do
  set -- $cfg
  echo "== requeue c=$1 deg>$2" >> gpurun_out/requeue.txt
  ATOS_PR_REQUEUE=$1 ATOS_PR_REQUEUE_DEG=$2 timeout 200 python tools/sweep.py pr --reps 3 --grid "512:512:1" >> gpurun_out/requeue.txt 2>&1
done
for cfg in "0 32" "10 32" "100 32"; do
  set -- $cfg
  echo "== C5 requeue c=$1 deg>$2" >> gpurun_out/requeue.txt
  ATOS_PR_REQUEUE=$1 ATOS_PR_REQUEUE_DEG=$2 timeout 300 python tools/sweep.py pr --scale 26 --reps 1 --grid "512:512:1" >> gpurun_out/requeue.txt 2>&1
done
ATOS_PR_REQUEUE=10 timeout 600 python -m pytest tests/test_gpu_pagerank.py -q -x > gpurun_out/t_pr_requeue.txt 2>&1
