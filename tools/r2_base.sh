set -x
mkdir -p gpurun_out/r2base
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nproc; grep -m1 "model name" /proc/cpuinfo
timeout 600 python bench.py --no-apps --no-cpu --no-bsp --steps 8 > gpurun_out/r2base/bench.json 2> gpurun_out/r2base/bench.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_relax_worker -c 1 -o gpurun_out/r2base/bfs_s26 python tools/run_app.py bfs scale=26 > gpurun_out/r2base/bfs_s26.log 2>&1
ls -la gpurun_out/r2base
