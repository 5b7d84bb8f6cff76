# full GPU check: all GPU tests, smoke, both benches, per-op ncu launch lists of both configs
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 1500 python -m pytest -q -m gpu tests -s > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_all.log
grep -E "passed|failed|Error|assert|rel L2" gpurun_out/pytest_all.log | tail -20
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout -s KILL 900 python bench.py --config rn50_mnv2 > gpurun_out/bench_cfg2.log 2>&1; tail -c 1200 gpurun_out/bench_cfg2.log
timeout -s KILL 900 python bench.py --config bert_rn50 --steps 200 > gpurun_out/bench_cfg3.log 2>&1; tail -c 2500 gpurun_out/bench_cfg3.log
CONFIG=bert_rn50 bash tools/ncu_times.sh
CONFIG=rn50_mnv2 CLIENTS=be bash tools/ncu_times.sh
du -sh gpurun_out
