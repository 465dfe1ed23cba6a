set -x
D=gpurun_out/r2next3
mkdir -p $D
timeout 1200 python tools/gc_order_study.py > $D/gc_order_study.txt 2>&1
M=launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active,launch__occupancy_limit_registers,launch__occupancy_limit_shared_mem,launch__occupancy_limit_warps,sm__maximum_warps_per_active_cycle_pct,launch__block_size,launch__grid_size,gpu__time_duration.sum
for spec in "worker=32 fetch_size=8 persistent=1" "worker=32 fetch_size=8 persistent=0" "worker=1024 fetch_size=128 persistent=1" "worker=1024 fetch_size=128 persistent=0"; do
  timeout 600 ncu --metrics $M --clock-control none -k regex:k_color -c 3 --csv python tools/run_app.py gc scale=20 ef=64 $spec > "$D/ncu_gc_$(echo $spec | tr ' =' '_-').csv" 2>&1
done
ls $D
