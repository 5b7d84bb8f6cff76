#!/bin/bash
# Kernel microbenchmarks (warm CUDA-event times at the BE / HP shapes) under routing / tuning variants,
# plus optional one-op ncu --set full capture (FOCUS=<op label>, FOCUS_CLIENT, CONFIG). Output: gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for what in ${MICRO:-wgs}; do
  echo "== $what default" >> gpurun_out/micro.txt
  timeout -s KILL 600 python tools/bench_kernels.py $what >> gpurun_out/micro.txt 2>&1
  for v in $VARIANTS; do
    echo "== $what $v" >> gpurun_out/micro.txt
    env $v timeout -s KILL 600 python tools/bench_kernels.py $what >> gpurun_out/micro.txt 2>&1
  done
done
if [ -n "$FOCUS" ]; then
  OURS='(gemm_|gemv_bt_kernel|conv_fwd_smallc|unary_kernel|binary_kernel|bn_|dw_|maxpool_kernel|maxpool_bwd_kernel|attention_kernel|layernorm_kernel|gelu_kernel|add_bf16_kernel|embed_kernel|col2im_kernel|ln_fwd_kernel|ln_bwd_kernel|attn_|avgpool|ce_kernel|mse_kernel|sgd_kernel|colsum_kernel|smallc_kernel|smallc2_kernel|wgs_kernel|atc_|cvf_kernel)'
  timeout -s KILL 900 ncu --set full --import-source on --clock-control none --kernel-name-base function -k "regex:$OURS" -c ${FOCUS_COUNT:-1} \
    -o gpurun_out/focus_${FOCUS//./_} python tools/profile/solo_runner.py --config ${CONFIG:-rn50_mnv2} --client ${FOCUS_CLIENT:-be} --only "$FOCUS" > gpurun_out/focus.log 2>&1
  ncu -i gpurun_out/focus_${FOCUS//./_}.ncu-rep --page details > gpurun_out/focus_${FOCUS//./_}.txt 2>&1
fi
cat gpurun_out/micro.txt
