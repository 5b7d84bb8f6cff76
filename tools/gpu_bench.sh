#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout 1200 python bench.py ${BENCH_ARGS} > gpurun_out/bench_${TAG:-main}.log 2>&1; echo "rc=$?" >> gpurun_out/bench_${TAG:-main}.log
tail -c 3000 gpurun_out/bench_${TAG:-main}.log
