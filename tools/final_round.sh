# End-of-round GPU pass: all GPU tests, smoke, the three benches, per-op ncu launch lists of every config.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout -s KILL 1500 python -m pytest -q -m gpu tests > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_all.log
tail -3 gpurun_out/pytest_all.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout -s KILL 900 python bench.py > gpurun_out/bench_cfg2.log 2>&1; tail -c 600 gpurun_out/bench_cfg2.log
timeout -s KILL 900 python bench.py --config bert_rn50 --steps 200 > gpurun_out/bench_cfg3.log 2>&1; tail -c 400 gpurun_out/bench_cfg3.log
timeout -s KILL 1200 python bench.py --config rn101_enc --steps 40 > gpurun_out/bench_cfg4.log 2>&1; tail -c 400 gpurun_out/bench_cfg4.log
timeout -s KILL 600 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_ref.log 2>&1; tail -c 300 gpurun_out/bench_ref.log
for c in rn50_mnv2 bert_rn50 rn101_enc; do CONFIG=$c bash tools/ncu_times.sh; done
du -sh gpurun_out
