"""Summarise the committed per-op ncu launch lists (profiles/<config>_<client>_ncu.csv) into one table
per config and client: device time per kernel family and the top launches with their DRAM GB/s."""
import csv
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main(out):
    lines = ["per-op device time (ncu gpu__time_duration.sum, --clock-control none, solo runner: tools/ncu_times.sh) "
             "per config and client"]
    for cfg in ("rn50_mnv2", "bert_rn50", "rn101_enc"):
        for c in ("hp", "be"):
            p = os.path.join(ROOT, "profiles", f"{cfg}_{c}_ncu.csv")
            if not os.path.exists(p):
                continue
            rows = list(csv.DictReader(open(p)))
            tot = sum(float(r["dur_ns"]) for r in rows)
            by = {}
            for r in rows:
                by[r["fn"]] = by.get(r["fn"], 0.0) + float(r["dur_ns"])
            lines.append(f"\n{cfg} {c}: {len(rows)} kernel ops, device sum {tot / 1e6:.3f} ms")
            for k, v in sorted(by.items(), key=lambda x: -x[1]):
                lines.append("   %-24s %8.3f ms %5.1f%%" % (k, v / 1e6, 100 * v / tot))
            for r in sorted(rows, key=lambda r: -float(r["dur_ns"]))[:10]:
                lines.append("      %-34s %-22s %8.1f us %6d GB/s grid %s" % (r["label"], r["fn"], float(r["dur_ns"]) / 1e3,
                                                                              float(r["dram_gbs"]), r["grid"]))
    open(out, "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r01", "ncu_launches_summary_all.txt"))
