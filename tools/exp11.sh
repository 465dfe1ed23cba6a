mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o gpurun_out/part2_full python tools/part_scan.py --scale 25 --parts 2 --apps bfs --reps 0 > gpurun_out/part2_full.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o gpurun_out/part1_full python tools/part_scan.py --scale 25 --parts 1 --apps bfs --reps 0 > gpurun_out/part1_full.log 2>&1
