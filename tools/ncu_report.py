"""Summarise .ncu-rep files (run here, no GPU): key throughput / traffic / stall metrics per kernel."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "lts__t_bytes.sum",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard", "smsp__inst_executed.sum"]


def report(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        print(path, "no rows")
        return []
    hdr = rows[0]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        res.append(d)
        name = d.get("Kernel Name", "")[:70]
        print(f"--- {name}")
        for k in KEYS:
            if k in d:
                print(f"   {k:70s} {d[k]}")
        stalls = {k: d[k] for k in d if k.startswith("smsp__average_warp_latency_issue_stalled") or k.startswith("smsp__pcsamp_warps_issue_stalled")}
        top = sorted(((float(v.replace(",", "")), k) for k, v in stalls.items() if v.replace(",", "").replace(".", "").isdigit()), reverse=True)[:6]
        for v, k in top:
            print(f"   stall {k:64s} {v}")
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        report(p)
