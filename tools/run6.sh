mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 1200 python -m pytest -q tests/test_config4_gpu.py tests/test_kernels_gpu.py -s -k "not batchnorm" > gpurun_out/pytest_cfg4.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_cfg4.log
grep -E "passed|failed|Error|assert|worst|encoder \(" gpurun_out/pytest_cfg4.log | tail -25
timeout -s KILL 1200 python bench.py --config rn101_enc --steps 40 > gpurun_out/bench_cfg4.log 2>&1; tail -c 3000 gpurun_out/bench_cfg4.log
CONFIG=rn101_enc bash tools/ncu_times.sh
CONFIG=bert_rn50 CLIENTS=be bash tools/ncu_times.sh
du -sh gpurun_out
