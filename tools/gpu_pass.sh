# GPU test pass: pytest -m gpu (all), smoke, one full bench line; outputs under gpurun_out/$1
set -x
D=gpurun_out/${1:-r2t}
mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" > $D/build.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q -x --durations=15 > $D/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> $D/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1
timeout 1200 python bench.py > $D/bench.json 2> $D/bench.err
tail -3 $D/pytest_gpu.log
