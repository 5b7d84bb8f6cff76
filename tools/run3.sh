# config-3 iteration: build, GPU tests, bench, focused ncu captures summarised on the box (reports deleted: 64 MiB cap)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 900 python -m pytest -q ${TESTS:-tests/test_kernels_bf16_gpu.py tests/test_kernels_gpu.py tests/test_e2e_config3_gpu.py tests/test_opcheck_config3_gpu.py} -s > gpurun_out/pytest_run3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_run3.log
grep -E "passed|failed|Error|assert|rel L2|worst" gpurun_out/pytest_run3.log | tail -30
if [ -z "$SKIP_BENCH" ]; then
timeout -s KILL 600 python bench.py --config bert_rn50 --steps 100 --warmup 5 --no-cpu-baseline > gpurun_out/bench_run3.log 2>&1
tail -c 2500 gpurun_out/bench_run3.log
fi
if [ -n "$FOCUS" ]; then
  CONFIG=${CONFIG:-bert_rn50} NCU_C=1 bash tools/ncu_focus.sh
  for f in gpurun_out/ncu_*.ncu-rep; do python tools/ncu_report.py $f > ${f%.ncu-rep}.txt 2>&1; done
  mkdir -p /tmp/ncurep; mv gpurun_out/*.ncu-rep /tmp/ncurep/ 2>/dev/null
  cat gpurun_out/ncu_*.txt | head -150
fi
if [ -n "$TIMES" ]; then CONFIG=bert_rn50 CLIENTS="$TIMES" bash tools/ncu_times.sh; fi
du -sh gpurun_out
