#!/bin/bash
# Full GPU pass: build, all GPU tests, smoke, default bench (config 2), per-op ncu tables of config 2
# with the profiler inputs. Output under gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
  timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
  timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
  tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log
fi
if [ -z "$SKIP_BENCH" ]; then
  timeout -s KILL 1500 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
  tail -c 600 gpurun_out/bench.log
fi
if [ -z "$SKIP_NCU" ]; then
  NCU_PROFILE=1 CLIENTS="${CLIENTS:-hp be}" bash tools/ncu_times.sh
  python tools/show_times.py ${CLIENTS:-hp be} > gpurun_out/show_times.txt 2>&1
  head -40 gpurun_out/show_times.txt
fi
