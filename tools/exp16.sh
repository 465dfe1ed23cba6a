mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_color.py -x -q > gpurun_out/t_color.txt 2>&1
: > gpurun_out/gc.txt
for v in default gcku8 gcku1; do
  L=$PWD/variants/libatos_$v.so; [ $v = default ] && L=$PWD/paper_conf_icpp_chenbpbyo22_b200/libatos.so
  echo "== $v" >> gpurun_out/gc.txt
  ATOS_LIB=$L timeout 200 python tools/sweep.py gc --reps 3 --grid "1024:128:1,512:128:1,512:64:1,256:128:1,1024:256:1" >> gpurun_out/gc.txt 2>&1
done
echo "== m5k4 pr" >> gpurun_out/gc.txt
ATOS_LIB=$PWD/variants/libatos_m5k4.so timeout 200 python tools/sweep.py pr --reps 3 --grid "256:256:1,256:128:1" >> gpurun_out/gc.txt 2>&1
echo "== m5k2 pr" >> gpurun_out/gc.txt
ATOS_LIB=$PWD/variants/libatos_m5k2.so timeout 200 python tools/sweep.py pr --reps 3 --grid "256:256:1" >> gpurun_out/gc.txt 2>&1
echo "== m5k2 road" >> gpurun_out/gc.txt
ATOS_LIB=$PWD/variants/libatos_m5k2.so timeout 200 python tools/sweep.py bfs-road --reps 2 --grid "256:256:1" >> gpurun_out/gc.txt 2>&1
echo "== default road" >> gpurun_out/gc.txt
timeout 200 python tools/sweep.py bfs-road --reps 2 --grid "256:256:1" >> gpurun_out/gc.txt 2>&1
