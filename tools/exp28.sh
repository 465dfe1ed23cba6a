mkdir -p gpurun_out
timeout 2400 compute-sanitizer --tool memcheck --print-limit 20 --error-exitcode 9 python -m pytest -x -q tests/test_gpu_bfs.py tests/test_gpu_pagerank.py tests/test_gpu_color.py tests/test_gpu_bsp.py > gpurun_out/memcheck_all.txt 2>&1
echo "rc=$?" >> gpurun_out/memcheck_all.txt
