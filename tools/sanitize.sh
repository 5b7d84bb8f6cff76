#!/bin/bash
# compute-sanitizer over one launch of every kernel family (tools/sanitize_kernels.py); summaries
# under gpurun_out/sanitize_<tool>.txt (copied to profiles/r02/ when committed).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for t in memcheck racecheck synccheck initcheck; do
  timeout -s KILL 900 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_kernels.py > gpurun_out/sanitize_$t.txt 2>&1
  echo "$t rc=$?" >> gpurun_out/sanitize_$t.txt
  tail -3 gpurun_out/sanitize_$t.txt
done
