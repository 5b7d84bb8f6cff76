#!/bin/bash
# Config-3 GPU round trip: build, the config-3 GPU tests, bench --config bert_rn50, per-op ncu launch lists.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout -s KILL 900 python -m pytest -x -q ${TESTS:-tests/test_kernels_bf16_gpu.py tests/test_opcheck_config3_gpu.py tests/test_e2e_config3_gpu.py} -s > gpurun_out/pytest_cfg3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_cfg3.log
tail -30 gpurun_out/pytest_cfg3.log
if [ -z "$SKIP_BENCH" ]; then
timeout -s KILL 900 python bench.py --config bert_rn50 --steps ${STEPS:-100} --warmup 5 > gpurun_out/bench_cfg3.log 2>&1; echo "rc=$?" >> gpurun_out/bench_cfg3.log
tail -c 3000 gpurun_out/bench_cfg3.log
fi
if [ -z "$SKIP_NCU" ]; then CONFIG=bert_rn50 bash tools/ncu_times.sh; fi
