#!/bin/bash
# ncu --set full on a few named ops (solo runner), reports under gpurun_out/
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
OURS='(gemm_|gemv_bt_kernel|conv_fwd_smallc|unary_kernel|binary_kernel|bn_|dw_|maxpool_kernel|maxpool_bwd_kernel|attention_kernel|layernorm_kernel|gelu_kernel|add_bf16_kernel|embed_kernel|col2im_kernel|ln_fwd_kernel|ln_bwd_kernel|attn_|avgpool|ce_kernel|mse_kernel|sgd_kernel|colsum_kernel|smallc_kernel|smallc2_kernel)'
for spec in $FOCUS; do
  client=${spec%%:*}; only=${spec#*:}
  tag=$(echo "$only" | tr -c 'a-zA-Z0-9\n' '_')
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k "regex:$OURS" -c ${NCU_C:-4} \
     -o gpurun_out/ncu_${client}_${tag} python tools/profile/solo_runner.py --config ${CONFIG:-rn50_mnv2} --client $client --only "$only" > gpurun_out/ncu_${client}_${tag}.out 2>&1
  echo "$spec rc=$?"
done
