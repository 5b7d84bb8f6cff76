"""Turn an `ncu --csv --page raw` metrics log of tools/profile/solo_runner.py into the profiler's
per-kernel_id CSV (sm_pct, mem_pct, dram_bytes, duration) + a time-share summary."""
import csv
import io
import sys


def parse(path):
    txt = open(path).read()
    start = txt.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(txt[start:])))
    out = {}
    for r in rows:
        try:
            i = int(r["ID"])
        except (KeyError, ValueError):
            continue
        d = out.setdefault(i, {"name": r.get("Kernel Name", "")})
        name, val = r.get("Metric Name"), r.get("Metric Value", "").replace(",", "")
        if name:
            try:
                d[name] = float(val)
            except ValueError:
                d[name] = val
    return [out[k] for k in sorted(out)]


def main(ncu_log, oplist, base, out_csv):
    launches = parse(ncu_log)
    ops = [l.rstrip("\n").split("\t") for l in open(oplist)]
    assert len(launches) == len(ops), (len(launches), len(ops))
    with open(out_csv, "w", newline="") as f:
        w = csv.writer(f)
        w.writerow(["kernel_id", "label", "fn", "dur_ns", "sm_pct", "mem_pct", "dram_bytes", "dram_gbs", "grid"])
        for (idx, fn, lab), m in zip(ops, launches):
            dur = m.get("gpu__time_duration.sum", 0.0)
            dram = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
            w.writerow([int(idx) + base, lab, fn, dur, m.get("sm__throughput.avg.pct_of_peak_sustained_elapsed", 0.0),
                        m.get("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", 0.0), dram,
                        dram / dur if dur else 0.0, m.get("launch__grid_size", 0)])


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4])
