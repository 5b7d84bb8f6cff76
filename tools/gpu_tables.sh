#!/bin/bash
# Per-op ncu tables (profiler inputs, NCU_PROFILE=1) of the given configs, plus optional tests first.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
if [ -n "$TESTS" ]; then
  timeout -s KILL ${TEST_TIMEOUT:-1200} python -m pytest $TESTS -q -x > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
  tail -3 gpurun_out/pytest_iter.log
fi
for cfg in ${CONFIGS:-bert_rn50 rn101_enc}; do
  CONFIG=$cfg NCU_PROFILE=1 CLIENTS="${CLIENTS:-hp be}" bash tools/ncu_times.sh
  CONFIG=$cfg python tools/show_times.py ${CLIENTS:-hp be} > gpurun_out/show_times_$cfg.txt 2>&1
  head -12 gpurun_out/show_times_$cfg.txt
done
