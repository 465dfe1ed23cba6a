mkdir -p gpurun_out
: > gpurun_out/pf.txt
for v in pf00 pf20 pf01 pf11 pf41; do
  echo "== $v" >> gpurun_out/pf.txt
  ATOS_LIB=$PWD/variants/libatos_$v.so timeout 200 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1,512:512:1" >> gpurun_out/pf.txt 2>&1
done
echo "== default" >> gpurun_out/pf.txt
timeout 200 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1,512:512:1,128:128:1" >> gpurun_out/pf.txt 2>&1
for v in pf00 default; do
  L=$PWD/variants/libatos_$v.so; [ $v = default ] && L=$PWD/paper_conf_icpp_chenbpbyo22_b200/libatos.so
  echo "== $v pr/mesh/gc" >> gpurun_out/pf.txt
  ATOS_LIB=$L timeout 200 python tools/sweep.py pr --reps 3 --grid "256:256:1,512:512:1" >> gpurun_out/pf.txt 2>&1
  ATOS_LIB=$L timeout 200 python tools/sweep.py bfs-mesh --reps 3 --grid "256:256:1" >> gpurun_out/pf.txt 2>&1
done
