#!/bin/bash
# Policy-knob sweep (PAPER §6.4 DUR_THRESHOLD sensitivity) + green-context BE partition.
# CONFIG (default rn50_mnv2), STEPS, and SWEEP (';'-separated bench flag sets) override the defaults.
mkdir -p gpurun_out/sweep
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
SWEEP=${SWEEP:-"--dur-ppm 10000;--dur-ppm 25000;--dur-ppm 50000;--dur-ppm 100000;--dur-ppm 25000 --be-partition 112;--dur-ppm 25000 --be-partition 72"}
IFS=';' read -ra CFGS <<< "$SWEEP"
for cfg in "${CFGS[@]}"; do
  tag=${CONFIG:-rn50_mnv2}_$(echo "$cfg" | tr -c 'a-z0-9\n' '_')
  timeout -s KILL 900 python bench.py --config ${CONFIG:-rn50_mnv2} --steps ${STEPS:-20} --warmup 3 --no-e2e --no-cpu-baseline --no-stress $cfg > gpurun_out/sweep/$tag.log 2>&1
  python - "$cfg" gpurun_out/sweep/$tag.log <<'PY'
import json, sys
line = [l for l in open(sys.argv[2]) if l.startswith("{")]
if not line: print(sys.argv[1], "FAILED"); sys.exit()
d = json.loads(line[-1])
print(f"{sys.argv[1]:36s} BE {d['value']:.2f} it/s ({d['be']['fraction_of_dedicated']:.3f} of ded)  HP p50 {d['hp']['p50_ms']:.3f} p99 {d['hp']['p99_ms']:.3f} ms  p99/ded {d['hp']['p99_vs_dedicated']:.3f}  p50/ded {d['hp']['p50_vs_dedicated']:.3f}")
PY
done | tee gpurun_out/sweep/summary_${CONFIG:-rn50_mnv2}.txt
