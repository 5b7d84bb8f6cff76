#!/bin/bash
# Max-pool / stem weight-gradient iteration: kernel tests, microbenchmarks, then config 3's bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_kernels_gpu.py tests/test_kernels_bf16_gpu.py tests/test_opcheck_config3_gpu.py -q -x 2>&1 | tail -3
timeout 300 python tools/bench_kernels.py pool
timeout 300 python tools/bench_kernels.py cwg 2>&1 | head -3
if [ -n "$BENCH3" ]; then
  timeout -s KILL 1500 python bench.py --config bert_rn50 --steps 20 --warmup 5 > gpurun_out/bench_bert_rn50.log 2>&1; echo "bench rc=$?"
  tail -c 300 gpurun_out/bench_bert_rn50.log
fi
