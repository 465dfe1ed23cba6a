mkdir -p gpurun_out
: > gpurun_out/big.txt
for ex in "big_chunk=2048" "big_chunk=4096" "big_chunk=8192" "big_chunk=16384" "big_threshold=16384" "big_threshold=65536" "big_threshold=16384,big_chunk=8192" "big_threshold=-1"; do
  echo "== $ex" >> gpurun_out/big.txt
  timeout 200 python tools/sweep.py bfs-rmat --reps 5 --grid "256:256:1" --extra $ex >> gpurun_out/big.txt 2>&1
done
