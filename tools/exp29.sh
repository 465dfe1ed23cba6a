mkdir -p gpurun_out
export ATOS_WATCHDOG_S=600
timeout 900 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 30 python tools/racecheck_small.py > gpurun_out/racecheck.txt 2>&1
echo "rc=$?" >> gpurun_out/racecheck.txt
