python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
echo "try_wait"; python tools/bench_gemm.py dbg
cd paper_conf_eurosys_stratimk24_b200/csrc && touch kernels/gemm.cu && make NVFLAGS_EXTRA=-DORION_MBAR_SPIN=1 > /dev/null 2>&1; cd ../..
echo "test_wait spin"; python tools/bench_gemm.py dbg
