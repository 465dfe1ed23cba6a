mkdir -p gpurun_out
: > gpurun_out/ku.txt
for v in t768k8 t768k6 t768k4 t640k8 t512k8; do
  echo "== $v" >> gpurun_out/ku.txt
  ATOS_LIB=$PWD/variants/libatos_$v.so timeout 200 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1,128:128:1,384:384:1" >> gpurun_out/ku.txt 2>&1
  ATOS_LIB=$PWD/variants/libatos_$v.so timeout 200 python tools/sweep.py pr --reps 3 --grid "256:256:1" >> gpurun_out/ku.txt 2>&1
done
echo "== default" >> gpurun_out/ku.txt
timeout 200 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1" >> gpurun_out/ku.txt 2>&1
