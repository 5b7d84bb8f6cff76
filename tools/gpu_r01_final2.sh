# End-of-round GPU pass on the committed tree: tests, smoke, configs 2-4 + reference arm, config-2
# per-op ncu launch lists, ncu --set full of the two BN backward kernels.
mkdir -p gpurun_out
md5sum paper_conf_eurosys_stratimk24_b200/csrc/kernels/*.cu > gpurun_out/src_md5.txt
bash tools/quick_check.sh
timeout -s KILL 900 python bench.py --config bert_rn50 --steps 200 > gpurun_out/bench_cfg3.log 2>&1; tail -c 300 gpurun_out/bench_cfg3.log
timeout -s KILL 600 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_ref.log 2>&1; tail -c 300 gpurun_out/bench_ref.log
CONFIG=rn50_mnv2 bash tools/ncu_times.sh
for k in bn_bwd_dx_kernel bn_bwd_reduce_kernel; do
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 6 -c 1 -o gpurun_out/full_$k python tools/profile/solo_runner.py --config rn50_mnv2 --client be > gpurun_out/ncu_full_$k.out 2>&1; echo ncu_full $k rc=$?
done
timeout -s KILL 1200 python bench.py --config rn101_enc --steps 40 > gpurun_out/bench_cfg4.log 2>&1; tail -c 300 gpurun_out/bench_cfg4.log
