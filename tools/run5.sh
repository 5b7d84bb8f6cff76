# config-4 + regression check: build, GPU tests (new + config 3), bench config 4, ncu lists of config 4
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 1200 python -m pytest -q -x tests/test_kernels_encoder_gpu.py tests/test_config4_gpu.py tests/test_e2e_config3_gpu.py tests/test_opcheck_config3_gpu.py -s > gpurun_out/pytest_cfg4.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_cfg4.log
grep -E "passed|failed|Error|assert|worst|encoder \(" gpurun_out/pytest_cfg4.log | tail -25
timeout -s KILL 1200 python bench.py --config rn101_enc --steps 40 > gpurun_out/bench_cfg4.log 2>&1; tail -c 3000 gpurun_out/bench_cfg4.log
CONFIG=rn101_enc bash tools/ncu_times.sh
du -sh gpurun_out
