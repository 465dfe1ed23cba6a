mkdir -p gpurun_out
: > gpurun_out/pr_sched.txt
for cfg in "0 0.5" "1e-2 0.85" "1e-2 0.5" "1e-3 0.5" "1e-4 0.25" "1e-1 0.7"; do
  set -- $cfg
  ATOS_PR_EPS0=$1 ATOS_PR_EPSF=$2 timeout 300 python tools/pr_sched.py --scale 22 >> gpurun_out/pr_sched.txt 2>&1
done
for cfg in "0 0.5" "1e-2 0.5" "1e-3 0.5"; do
  set -- $cfg
  ATOS_PR_EPS0=$1 ATOS_PR_EPSF=$2 timeout 300 python tools/pr_sched.py --scale 26 --seed 5 --reps 1 >> gpurun_out/pr_sched.txt 2>&1
done
