"""Turn an `ncu --csv --page raw` metrics log of tools/profile/solo_runner.py into the profiler's
per-kernel_id CSV (sm_pct, mem_pct, dram_bytes, duration) + a time-share summary."""
import csv
import io
import sys


def parse(path):
    """ncu --csv --page raw: one row per launch, metric names as columns (second row = units)."""
    txt = open(path).read()
    start = txt.find('"ID"')
    rows = list(csv.reader(io.StringIO(txt[start:])))
    hdr = rows[0]
    out = []
    for r in rows[1:]:
        if not r or not r[0].isdigit():
            continue   # units row
        d = {"name": r[hdr.index("Kernel Name")]}
        for k, v in zip(hdr, r):
            try:
                d[k] = float(v.replace(",", ""))
            except ValueError:
                pass
        out.append(d)
    return out


# the profiler's further inputs (P:838-847 throughputs, P:859-870 occupancy limits): CSV column <- ncu metric
EXTRA = [("tc_pct", "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed"),
         ("tensor_pct", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"),
         ("fma_pct", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_elapsed"),
         ("block", "launch__block_size"), ("regs", "launch__registers_per_thread"),
         ("occ_blocks", "launch__occupancy_limit_blocks"), ("occ_regs", "launch__occupancy_limit_registers"),
         ("occ_smem", "launch__occupancy_limit_shared_mem"), ("occ_warps", "launch__occupancy_limit_warps"),
         ("smem_dyn", "launch__shared_mem_per_block_dynamic"), ("smem_static", "launch__shared_mem_per_block_static")]


def main(ncu_log, oplist, base, out_csv):
    raw = parse(ncu_log)
    ops = [l.rstrip("\n").split("\t") for l in open(oplist)]
    # an op may issue several kernels (4th oplist column): sum their durations / bytes, keep the
    # first kernel's grid and counters (the op's main kernel)
    launches, i = [], 0
    for op in ops:
        k = int(op[3]) if len(op) > 3 else 1
        group = raw[i:i + k]
        i += k
        m = dict(group[0]) if group else {}
        for extra in group[1:]:
            for key in ("gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum"):
                m[key] = m.get(key, 0.0) + extra.get(key, 0.0)
        launches.append(m)
    assert i == len(raw), (i, len(raw))
    ops = [op[:3] for op in ops]
    with open(out_csv, "w", newline="") as f:
        w = csv.writer(f)
        w.writerow(["kernel_id", "label", "fn", "dur_ns", "sm_pct", "mem_pct", "dram_bytes", "dram_gbs", "grid"] +
                   [c for c, _ in EXTRA])
        for (idx, fn, lab), m in zip(ops, launches):
            dur = m.get("gpu__time_duration.sum", 0.0)
            dram = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
            w.writerow([int(idx) + base, lab, fn, dur, m.get("sm__throughput.avg.pct_of_peak_sustained_elapsed", 0.0),
                        m.get("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", 0.0), dram,
                        dram / dur if dur else 0.0, m.get("launch__grid_size", 0)] + [m.get(k, "") for _, k in EXTRA])


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4])
