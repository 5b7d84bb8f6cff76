mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -s KILL 600 python -m pytest -q -m gpu tests/test_kernels_gpu.py > gpurun_out/pytest_k.log 2>&1; tail -2 gpurun_out/pytest_k.log
CONFIG=rn50_mnv2 CLIENTS=be bash tools/ncu_times.sh
