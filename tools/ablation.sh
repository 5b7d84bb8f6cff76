#!/bin/bash
# Policy ablation (PAPER Fig. 14) on BASELINE config 2 (or $CONFIG): one bench line per policy.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for pol in ${POLICIES:-streams priorities profiles orion orion_noprio}; do
  timeout -s KILL 900 python bench.py --config ${CONFIG:-rn50_mnv2} --policy $pol --steps ${STEPS:-20} --warmup 5 --no-e2e --no-cpu-baseline --no-stress \
    > gpurun_out/ablation_${CONFIG:-rn50_mnv2}_$pol.log 2>&1
  python - "$pol" "gpurun_out/ablation_${CONFIG:-rn50_mnv2}_$pol.log" <<'PY'
import json, sys
line = [l for l in open(sys.argv[2]) if l.startswith('{"metric"')]
if not line:
    print(sys.argv[1], "FAILED"); sys.exit()
d = json.loads(line[-1])
print(f"{sys.argv[1]:14s} HP p50 {d['hp']['p50_ms']:.3f} ms p99 {d['hp']['p99_ms']:.3f} ms (x{d['hp']['p99_vs_dedicated']:.3f} of dedicated {d['hp']['dedicated_p99_ms']:.3f})"
      f"  BE {d['be']['collocated_its']:.2f} it/s ({d['be']['fraction_of_dedicated']:.3f} of dedicated)")
PY
done | tee gpurun_out/ablation_${CONFIG:-rn50_mnv2}.txt
