python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for d in 0 1 2 4 3 7; do echo "dbg=$d"; ORION_TCM_DEBUG=$d python tools/bench_gemm.py dbg; done
