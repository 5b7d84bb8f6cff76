bash tools/quick_check.sh
timeout -s KILL 900 python bench.py --config bert_rn50 --steps 200 > gpurun_out/bench_cfg3.log 2>&1; tail -c 300 gpurun_out/bench_cfg3.log
CONFIG=rn50_mnv2 bash tools/ncu_times.sh
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:bn_bwd_dx_kernel -s 20 -c 1 -o gpurun_out/bwd_dx_full python tools/profile/solo_runner.py --config rn50_mnv2 --client be > gpurun_out/ncu_full.out 2>&1; echo ncu_full rc=$?
