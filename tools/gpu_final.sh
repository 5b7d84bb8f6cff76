#!/bin/bash
# End-of-round GPU pass: build, all GPU tests, smoke, BN statistics A/B, default bench (config 2),
# config-2 per-op ncu tables with the profiler inputs, one ncu --set full of the dominant BE kernels.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log
if [ -n "$BN_AB" ]; then
  for u in 8 16 8 16; do echo "== BN_STATS_U $u"; ORION_BN_STATS_U=$u timeout 300 python tools/bench_kernels.py bn | tail -13; done > gpurun_out/bn_ab.txt 2>&1
  grep -E "==|total" gpurun_out/bn_ab.txt
fi
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/clocks_before.csv 2>&1
timeout -s KILL 1500 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
tail -c 400 gpurun_out/bench.log
if [ -z "$SKIP_NCU" ]; then
  NCU_PROFILE=1 CLIENTS="hp be" bash tools/ncu_times.sh
  python tools/show_times.py hp be > gpurun_out/show_times.txt 2>&1
  head -30 gpurun_out/show_times.txt
  OURS='(gemm_|bn_|dw_|wgs_kernel|atc_|cvf_kernel|unary_kernel|binary_kernel)'
  for lab in features.2.expand_bn.relu6_bwd features.2.expand.wgrad; do
    timeout -s KILL 600 ncu --set full --import-source on --clock-control none --kernel-name-base function -k "regex:$OURS" -c 1 \
      -o gpurun_out/full_${lab//./_} python tools/profile/solo_runner.py --config rn50_mnv2 --client be --only "$lab" > /dev/null 2>&1
    ncu -i gpurun_out/full_${lab//./_}.ncu-rep --page details > gpurun_out/full_${lab//./_}.txt 2>&1
  done
fi
