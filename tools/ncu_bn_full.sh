# ncu --set full of the dominant BE kernels of config 2 (MobileNetV2 features.2 expand BN backward:
# the 49th bn_bwd_reduce / bn_bwd_dx launch of one solo BE iteration).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for k in bn_bwd_dx_kernel bn_bwd_reduce_kernel; do
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 48 -c 1 -o gpurun_out/full48_$k python tools/profile/solo_runner.py --config rn50_mnv2 --client be > gpurun_out/ncu_full48_$k.out 2>&1; echo ncu_full $k rc=$?
done
