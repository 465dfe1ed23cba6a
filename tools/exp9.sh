mkdir -p gpurun_out
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,smsp__inst_executed.sum,l1tex__data_pipe_lsu_wavefronts.sum,l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum,sm__warps_active.avg.pct_of_peak_sustained_active
timeout 600 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 4 --csv python tools/part_scan.py --parts 2 --apps bfs --reps 0 > gpurun_out/ncu_part2.csv 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:k_relax_worker -c 1 --csv python tools/part_scan.py --parts 1 --apps bfs --reps 0 > gpurun_out/ncu_part1.csv 2>&1
