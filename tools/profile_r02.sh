#!/bin/bash
# Round-2 profiling pass over the current build (run under gpurun from the repo root); writes gpurun_out/r02prof/.
# 1. the bench line (not under a profiler); 2. per-launch DRAM traffic of the BFS (C5), PageRank (C3, C5) and
# colouring (C4) workers; 3. ncu --set full (+ source) of the BFS worker at C5 and the PageRank worker at C3;
# 4. the launch list of a short bench run (cold-cache, serialised: compare shares, not absolutes).
set -x
D=gpurun_out/r02prof
mkdir -p $D
timeout 1500 python bench.py > $D/bench.json 2> $D/bench.err
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 300 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/run_app.py bfs scale=26 > $D/bfs_s26_traffic.csv 2>&1
timeout 300 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/run_app.py pr scale=22 > $D/pr_s22_traffic.csv 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/run_app.py pr scale=26 seed=5 > $D/pr_s26_traffic.csv 2>&1
timeout 300 ncu --metrics $M --clock-control none -k regex:k_color_cta -c 1 --csv python tools/run_app.py gc scale=20 ef=64 > $D/gc_s20_traffic.csv 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o $D/bfs_s26_full python tools/run_app.py bfs scale=26 > $D/bfs_s26_full.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o $D/pr_s22_full python tools/run_app.py pr scale=22 > $D/pr_s22_full.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:^k_ -c 400 --csv --log-file $D/bench_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-apps --no-bsp > $D/bench_ncu.log 2>&1
ls -la $D
