mkdir -p gpurun_out
: > gpurun_out/gate.txt
for v in gate0 default; do
  L=$PWD/variants/libatos_$v.so; [ $v = default ] && L=$PWD/paper_conf_icpp_chenbpbyo22_b200/libatos.so
  echo "== $v" >> gpurun_out/gate.txt
  ATOS_LIB=$L timeout 200 python tools/sweep.py bfs-mesh --reps 3 --grid "256:256:1,32:8:1" >> gpurun_out/gate.txt 2>&1
  ATOS_LIB=$L timeout 200 python tools/sweep.py bfs-road --reps 3 --grid "256:256:1" >> gpurun_out/gate.txt 2>&1
  ATOS_LIB=$L timeout 200 python tools/sweep.py bfs-rmat --reps 3 --grid "256:256:1" >> gpurun_out/gate.txt 2>&1
  ATOS_LIB=$L timeout 200 python tools/sweep.py pr --reps 3 --grid "512:512:1" >> gpurun_out/gate.txt 2>&1
  ATOS_LIB=$L timeout 200 python tools/sweep.py gc --reps 3 --grid "1024:128:1" >> gpurun_out/gate.txt 2>&1
done
