"""Summarise an ncu --set full report: key SOL / occupancy metrics and the top stalled SASS lines."""
import csv, io, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
r = csv.reader(io.StringIO(out)); h = next(r)
keys = ["duration", "elapsed cycles", "dram throughput", "memory throughput", "compute (sm) throughput", "registers",
        "achieved occupancy", "l2 cache throughput", "l1/tex cache throughput", "issue slots busy", "executed ipc active",
        "warp cycles per issued", "shared memory configuration size", "dynamic shared memory"]
for row in r:
    d = dict(zip(h, row))
    n = d.get("Metric Name", "")
    if any(k in n.lower() for k in keys):
        print(f"{d.get('Section Name')} | {n} | {d.get('Metric Value')} {d.get('Metric Unit')}")
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = 1 if rows and rows[0] and rows[0][0] == "Kernel Name" else 0
h = rows[hi]; idx = {k: i for i, k in enumerate(h)}
key = "Warp Stall Sampling (All Samples)"
data = []
for row in rows[hi + 1:]:
    if len(row) < len(h):
        continue
    try:
        v = float(row[idx[key]] or 0)
    except ValueError:
        continue
    data.append((v, row[idx["Address"]], row[idx["Source"]]))
tot = sum(d[0] for d in data) or 1
print("stall samples", tot)
for d in sorted(data, reverse=True)[:top]:
    print("%6.1f%%" % (100 * d[0] / tot), d[1][-5:], d[2][:110])
