"""Print the per-op device-time summary written by tools/ncu_times.sh."""
import collections
import csv
import os
import sys

for c in (sys.argv[1:] or ["hp", "be"]):
    rows = list(csv.DictReader(open(f"gpurun_out/times_{os.environ.get('CONFIG', 'rn50_mnv2')}_{c}.csv")))
    tot = sum(float(r["dur_ns"]) for r in rows)
    by = collections.defaultdict(float)
    for r in rows:
        by[r["fn"]] += float(r["dur_ns"])
    print(c, len(rows), "ops, device sum %.3f ms" % (tot / 1e6))
    for k, v in sorted(by.items(), key=lambda x: -x[1])[:12]:
        print("   %-14s %8.3f ms %5.1f%%" % (k, v / 1e6, 100 * v / tot))
    for r in sorted(rows, key=lambda r: -float(r["dur_ns"]))[:16]:
        print("     ", r["label"], r["fn"], "%.1f us" % (float(r["dur_ns"]) / 1e3), "%.0f GB/s" % float(r["dram_gbs"]))
