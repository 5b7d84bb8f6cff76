#!/bin/bash
# Benches of configs 3 / 4 / inf-inf on the current tree + the config-4 HP per-op ncu table.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for c in ${BCONFIGS:-bert_rn50 rn101_enc infinf}; do
  timeout -s KILL 1500 python bench.py --config $c --steps 20 --warmup 5 > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  tail -c 400 gpurun_out/bench_$c.log; echo
done
if [ -n "$HP_TABLE" ]; then
  CONFIG=rn101_enc NCU_PROFILE=1 NCU_TIMEOUT=2400 CLIENTS=hp bash tools/ncu_times.sh
  CONFIG=rn101_enc python tools/show_times.py hp > gpurun_out/show_times_rn101_enc_hp.txt 2>&1; head -12 gpurun_out/show_times_rn101_enc_hp.txt
fi
