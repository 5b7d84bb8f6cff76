#!/bin/bash
# Full GPU round trip: build, GPU tests, smoke, bench (with CPU baseline), ncu launch list of the
# hot path, per-op ncu counters of both clients, one full ncu capture of the top BE kernel.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
timeout 1200 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "rc=$?" >> gpurun_out/bench.log
if [ -z "$SKIP_NCU" ]; then
OURS='(gemm_kernel|gemm_tc_kernel|gemm_atb_kernel|gemm_rows_kernel|gemv_bt_kernel|unary_kernel|binary_kernel|bn_|dw_|maxpool_kernel|avgpool|ce_kernel|mse_kernel|sgd_kernel|colsum_kernel)'
M=gpu__time_duration.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size
for c in hp be; do
  timeout 1200 ncu --metrics $M --clock-control none --csv --page raw --kernel-name-base function -k "regex:$OURS" --log-file gpurun_out/ncu_${c}.csv python tools/profile/solo_runner.py --client $c > gpurun_out/ncu_${c}.out 2>&1
done
python tools/profile/ncu_summarize.py gpurun_out/ncu_hp.csv gpurun_out/oplist_rn50_mnv2_hp.txt 0 gpurun_out/rn50_mnv2_hp_ncu.csv > gpurun_out/ncu_sum.log 2>&1
python tools/profile/ncu_summarize.py gpurun_out/ncu_be.csv gpurun_out/oplist_rn50_mnv2_be.txt 10000 gpurun_out/rn50_mnv2_be_ncu.csv >> gpurun_out/ncu_sum.log 2>&1
if [ -n "$TOP" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function -k "regex:$OURS" -c 1 -o gpurun_out/top_kernel python tools/profile/solo_runner.py --client be --only "$TOP" > gpurun_out/ncu_top.out 2>&1
fi
fi
tail -c 1500 gpurun_out/bench.log
