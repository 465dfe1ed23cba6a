#!/bin/bash
# One profiling pass over the current build (run under gpurun from the repo root); writes gpurun_out/prof_*.
# 1. bench line (not under a profiler); 2. per-launch DRAM traffic of the BFS (C5), PageRank (C3 and C5) and
# colouring (C4) workers; 3. ncu --set full of the BFS worker at S25 and the PageRank worker at S22;
# 4. the bench's launch list.
set -x
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/prof_bench.json 2> gpurun_out/prof_bench.err
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum
timeout 300 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/run_app.py bfs scale=26 > gpurun_out/prof_bfs_s26_traffic.csv 2>&1
timeout 300 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/run_app.py pr scale=22 > gpurun_out/prof_pr_s22_traffic.csv 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/run_app.py pr scale=26 seed=5 > gpurun_out/prof_pr_s26_traffic.csv 2>&1
timeout 300 ncu --metrics $M --clock-control none -k regex:k_color_cta -c 1 --csv python tools/run_app.py gc scale=20 ef=64 > gpurun_out/prof_gc_s20_traffic.csv 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o gpurun_out/prof_bfs_s25 python tools/run_app.py bfs scale=25 > gpurun_out/prof_bfs_s25.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o gpurun_out/prof_pr_s22 python tools/run_app.py pr scale=22 > gpurun_out/prof_pr_s22.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:^k_ -c 3000 --csv --log-file gpurun_out/prof_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu > gpurun_out/prof_bench_ncu.log 2>&1
ls -la gpurun_out
