#!/bin/bash
# Per-launch device time of every op of one client (solo runner), under ncu (serialised, cold-ish caches).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
OURS='(gemm_|gemv_bt_kernel|conv_fwd_smallc|unary_kernel|binary_kernel|bn_|dw_|maxpool_kernel|maxpool_bwd_kernel|attention_kernel|layernorm_kernel|gelu_kernel|add_bf16_kernel|embed_kernel|col2im_kernel|ln_fwd_kernel|ln_bwd_kernel|attn_|avgpool|ce_kernel|mse_kernel|sgd_kernel|colsum_kernel|smallc_kernel|smallc2_kernel|wgs_kernel|atc_|cvf_kernel)'
# quick pass (device time + DRAM bytes) by default; NCU_PROFILE=1 adds the profiler's inputs
# (P:838-847 throughputs, tensor / FMA pipe activity, P:859-870 occupancy limits)
METRICS=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size
if [ -n "$NCU_PROFILE" ]; then
  METRICS=$METRICS,launch__block_size,sm__throughput.avg.pct_of_peak_sustained_elapsed,gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_elapsed,launch__occupancy_limit_blocks,launch__occupancy_limit_registers,launch__occupancy_limit_shared_mem,launch__occupancy_limit_warps,launch__registers_per_thread,launch__shared_mem_per_block_dynamic,launch__shared_mem_per_block_static
fi
for c in ${CLIENTS:-hp be}; do
  timeout -s KILL ${NCU_TIMEOUT:-900} ncu --metrics $METRICS --clock-control none --csv --page raw \
     --kernel-name-base function -k "regex:$OURS" --log-file gpurun_out/ncu_times_${CONFIG:-rn50_mnv2}_${c}.csv python tools/profile/solo_runner.py --config ${CONFIG:-rn50_mnv2} --client $c > gpurun_out/ncu_times_${CONFIG:-rn50_mnv2}_${c}.out 2>&1
  base=0; [ "$c" = be ] && base=10000
  python tools/profile/ncu_summarize.py gpurun_out/ncu_times_${CONFIG:-rn50_mnv2}_${c}.csv gpurun_out/oplist_${CONFIG:-rn50_mnv2}_${c}.txt 0 gpurun_out/times_${CONFIG:-rn50_mnv2}_${c}.csv
  python tools/profile/ncu_summarize.py gpurun_out/ncu_times_${CONFIG:-rn50_mnv2}_${c}.csv gpurun_out/oplist_${CONFIG:-rn50_mnv2}_${c}.txt $base gpurun_out/${CONFIG:-rn50_mnv2}_${c}_ncu.csv
done
