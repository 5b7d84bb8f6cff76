#!/bin/bash
# ncu --set full captures of the ops named in $LABELS (solo runner, first matching launch each),
# summarised as text under gpurun_out/focus_<label>.txt; optional pytest selection in $TESTS first.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
if [ -n "$TESTS" ]; then
  timeout -s KILL ${TEST_TIMEOUT:-1500} python -m pytest $TESTS -q -x ${PYTEST_ARGS} > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
  tail -5 gpurun_out/pytest_iter.log
fi
OURS='(gemm_|gemv_bt_kernel|conv_fwd_smallc|unary_kernel|binary_kernel|bn_|dw_|maxpool_kernel|maxpool_bwd_kernel|attention_kernel|layernorm_kernel|gelu_kernel|add_bf16_kernel|embed_kernel|col2im_kernel|ln_fwd_kernel|ln_bwd_kernel|attn_|avgpool|ce_kernel|mse_kernel|sgd_kernel|colsum_kernel|smallc_kernel|smallc2_kernel|wgs_kernel|atc_|cvf_kernel)'
for L in $LABELS; do
  f=gpurun_out/focus_${L//./_}
  timeout -s KILL 600 ncu --set full --import-source on --clock-control none --kernel-name-base function -k "regex:$OURS" -c ${FOCUS_COUNT:-1} \
    -o $f python tools/profile/solo_runner.py --config ${CONFIG:-rn50_mnv2} --client ${FOCUS_CLIENT:-be} --only "$L" > $f.log 2>&1
  ncu -i $f.ncu-rep --page details > $f.txt 2>&1
  grep -E "Duration|DRAM Throughput|Registers Per|Achieved Occupancy|Executed Ipc A|Issue Slots Busy" $f.txt | head -8
done
