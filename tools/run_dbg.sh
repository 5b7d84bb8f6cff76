python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for d in 0 1 2 4 8 9 15 14; do echo "dbg=$d"; ORION_TMK_DEBUG=$d python tools/bench_gemm.py dbg; done
