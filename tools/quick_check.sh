# GPU pass on the current tree: GPU tests, smoke, config-2 bench (uses MEASURED_PEAKS.json).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 1200 python -m pytest -q -m gpu tests > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_all.log
tail -3 gpurun_out/pytest_all.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout -s KILL 900 python bench.py > gpurun_out/bench_cfg2.log 2>&1; tail -c 600 gpurun_out/bench_cfg2.log
