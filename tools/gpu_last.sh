#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout -s KILL 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log
timeout -s KILL 1500 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
timeout -s KILL 1500 python bench.py --config bert_rn50 --steps 20 --warmup 5 > gpurun_out/bench_bert_rn50.log 2>&1; echo "bench3 rc=$?"
CONFIG=bert_rn50 NCU_PROFILE=1 CLIENTS=be bash tools/ncu_times.sh
CONFIG=bert_rn50 python tools/show_times.py be > gpurun_out/show_times_bert_rn50_be.txt 2>&1; head -12 gpurun_out/show_times_bert_rn50_be.txt
