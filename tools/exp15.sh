mkdir -p gpurun_out
: > gpurun_out/occ.txt
for v in m5k4 m5k2 m6k2; do
  echo "== $v" >> gpurun_out/occ.txt
  ATOS_LIB=$PWD/variants/libatos_$v.so timeout 200 python tools/sweep.py bfs-rmat --reps 3 --grid "256:256:1" >> gpurun_out/occ.txt 2>&1
  ATOS_LIB=$PWD/variants/libatos_$v.so timeout 200 python tools/sweep.py bfs-mesh --reps 2 --grid "256:256:1" >> gpurun_out/occ.txt 2>&1
done
