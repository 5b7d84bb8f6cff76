mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
CLIENTS="${CLIENTS:-be}" bash tools/ncu_times.sh
python tools/show_times.py ${CLIENTS:-be} > gpurun_out/show_times.txt 2>&1
timeout 900 python bench.py --steps 100 --warmup 3 --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
tail -3 gpurun_out/pytest_gpu.log; head -40 gpurun_out/show_times.txt; tail -c 1200 gpurun_out/bench.log
