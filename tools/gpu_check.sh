#!/bin/bash
# One GPU round-trip: build, GPU tests, smoke, short benches. Output under gpurun_out/.
set -x
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py --config toy --steps 200 --warmup 3 --no-cpu-baseline > gpurun_out/bench_toy.log 2>&1; echo "rc=$?" >> gpurun_out/bench_toy.log
tail -5 gpurun_out/pytest_gpu.log
