#!/bin/bash
# Full GPU round trip: build, GPU tests, smoke, bench (with CPU baseline), per-op device times of both
# clients under ncu (launch list), optional full ncu capture of named ops. Output under gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/clocks_before.csv 2>&1
timeout -s KILL 1500 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "rc=$?" >> gpurun_out/bench.log
if [ -z "$SKIP_NCU" ]; then
  bash tools/ncu_times.sh
  if [ -n "$FOCUS" ]; then bash tools/ncu_focus.sh; fi
fi
tail -c 1500 gpurun_out/bench.log
