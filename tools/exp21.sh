mkdir -p gpurun_out
timeout 1500 compute-sanitizer --tool memcheck --print-limit 20 --error-exitcode 9 python -m pytest -x -q tests/test_gpu_partitioned.py "tests/test_gpu_bfs.py::test_layout_modes" "tests/test_gpu_color.py::test_layout_modes_valid" "tests/test_gpu_pagerank.py::test_layout_input_and_auto_agree" "tests/test_gpu_bfs.py::test_layout_degree_mesh_closed_form" > gpurun_out/memcheck.txt 2>&1
echo "rc=$?" >> gpurun_out/memcheck.txt
