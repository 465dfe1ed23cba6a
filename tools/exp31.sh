mkdir -p gpurun_out
: > gpurun_out/layout_apps.txt
for L in input degree; do
  echo "== $L" >> gpurun_out/layout_apps.txt
  timeout 200 python tools/sweep.py gc --reps 3 --grid "1024:128:1" --layout $L >> gpurun_out/layout_apps.txt 2>&1
  timeout 200 python tools/sweep.py pr --reps 3 --grid "512:512:1" --layout $L >> gpurun_out/layout_apps.txt 2>&1
  timeout 200 python tools/sweep.py bfs-rmat --scale 22 --reps 5 --grid "256:256:1" --layout $L >> gpurun_out/layout_apps.txt 2>&1
  timeout 200 python tools/sweep.py bfs-mesh --reps 2 --grid "256:256:1" --layout $L >> gpurun_out/layout_apps.txt 2>&1
done
