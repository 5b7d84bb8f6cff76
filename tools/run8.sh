mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 1500 python -m pytest -q -m gpu tests -s > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_all.log
grep -E "passed|failed|Error|assert" gpurun_out/pytest_all.log | tail -12
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout -s KILL 900 python bench.py > gpurun_out/bench_cfg2.log 2>&1; tail -c 1600 gpurun_out/bench_cfg2.log
timeout -s KILL 900 python bench.py --config bert_rn50 --steps 200 > gpurun_out/bench_cfg3.log 2>&1; tail -c 1600 gpurun_out/bench_cfg3.log
CONFIG=rn50_mnv2 bash tools/ncu_times.sh
CONFIG=rn101_enc bash tools/ncu_times.sh
du -sh gpurun_out
