#!/bin/bash
# Kernel-level iteration: build, the kernel GPU tests (KT_TESTS), microbenchmarks (KT_MICRO).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest ${KT_TESTS:-tests/test_kernels_gpu.py tests/test_kernels_encoder_gpu.py} -q -x 2>&1 | tail -5
for m in ${KT_MICRO:-dw stem attn}; do timeout 300 python tools/bench_kernels.py $m; done
