mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -50 gpurun_out/build.log; exit 1; }
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gemm_tcm -c 1 -o gpurun_out/tcm_stream -f python tools/one_gemm.py ${SHAPE:-1204224 96 16 2} > gpurun_out/ncu_tcm.log 2>&1
tail -n 3 gpurun_out/ncu_tcm.log
