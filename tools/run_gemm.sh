mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_kernels_gpu.py -x -q -k "gemm" > gpurun_out/pytest_gemm.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gemm.log
tail -15 gpurun_out/pytest_gemm.log
timeout 300 python tools/bench_gemm.py generic mnv2 > gpurun_out/bench_gemm.txt 2>&1
cat gpurun_out/bench_gemm.txt
