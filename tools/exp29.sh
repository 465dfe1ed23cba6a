mkdir -p gpurun_out
timeout 2400 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 30 python -m pytest -x -q "tests/test_gpu_bfs.py::test_small_named" "tests/test_gpu_bfs.py::test_mesh_road_percolated" "tests/test_gpu_color.py::test_named" "tests/test_gpu_pagerank.py::test_star_closed_form" > gpurun_out/racecheck.txt 2>&1
echo "rc=$?" >> gpurun_out/racecheck.txt
