mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
python tools/bench_ops.py > gpurun_out/bench_ops.txt 2>&1
python tools/bench_gemm.py > gpurun_out/bench_gemm.txt 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:bn_stats -c 1 -s 2 -o gpurun_out/bn_stats_small -f python tools/bench_ops.py bn 18816 64 > gpurun_out/ncu_bn.log 2>&1
cat gpurun_out/bench_ops.txt gpurun_out/bench_gemm.txt
