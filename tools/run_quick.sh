mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
CLIENTS=be bash tools/ncu_times.sh
python tools/show_times.py be > gpurun_out/show_be.txt 2>&1
tail -3 gpurun_out/pytest_gpu.log; head -30 gpurun_out/show_be.txt
