#!/bin/bash
# One build -> test -> measure iteration on the GPU box (used through gpurun):
#   TESTS="tests/x.py ..."  pytest selection (default: none)
#   CLIENTS="be hp"         per-op ncu launch lists of those clients (CONFIG, default rn50_mnv2; none if empty)
#   BENCH_ARGS="..."        run bench.py with these args when set
#   FOCUS="label" / FOCUS_CLIENT   one `ncu --set full` capture of the op with that label
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
nproc > gpurun_out/nproc.txt
if [ -n "$TESTS" ]; then
  timeout -s KILL ${TEST_TIMEOUT:-1200} python -m pytest $TESTS -q -x ${PYTEST_ARGS} > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
  tail -5 gpurun_out/pytest_iter.log
fi
if [ -n "$CLIENTS" ]; then
  CLIENTS="$CLIENTS" bash tools/ncu_times.sh
  python tools/show_times.py $CLIENTS > gpurun_out/show_times.txt 2>&1
  head -60 gpurun_out/show_times.txt
fi
if [ -n "$FOCUS" ]; then
  OURS='(gemm_|gemv_bt_kernel|conv_fwd_smallc|unary_kernel|binary_kernel|bn_|dw_|maxpool_kernel|maxpool_bwd_kernel|attention_kernel|layernorm_kernel|gelu_kernel|add_bf16_kernel|embed_kernel|col2im_kernel|ln_fwd_kernel|ln_bwd_kernel|attn_|avgpool|ce_kernel|mse_kernel|sgd_kernel|colsum_kernel|smallc_kernel|smallc2_kernel|wgs_kernel|atc_|cvf_kernel)'
  timeout -s KILL 600 ncu --set full --import-source on --clock-control none --kernel-name-base function -k "regex:$OURS" -c ${FOCUS_COUNT:-1} \
    -o gpurun_out/focus_${FOCUS//./_} python tools/profile/solo_runner.py --config ${CONFIG:-rn50_mnv2} --client ${FOCUS_CLIENT:-be} --only "$FOCUS" > gpurun_out/focus.log 2>&1
  ncu -i gpurun_out/focus_${FOCUS//./_}.ncu-rep --page details > gpurun_out/focus_${FOCUS//./_}.txt 2>&1
fi
if [ -n "$BENCH_ARGS" ]; then
  timeout -s KILL 1500 python bench.py $BENCH_ARGS > gpurun_out/bench_iter.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_iter.log
  tail -c 2500 gpurun_out/bench_iter.log
fi
