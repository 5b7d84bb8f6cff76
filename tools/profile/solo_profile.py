"""Offline profiler driver (§5.2): solo per-op profile of each client of a config ->
profiles/<config>_<client>.csv (kernel_id, label, fn, cls, sm_needed, dur_ns, flops, bytes, source),
plus a top-N summary by time share. Run on the GPU box."""
import argparse
import collections
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import profiler as PR  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="rn50_mnv2")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles"))
    ap.add_argument("--top", type=int, default=25)
    ap.add_argument("--ncu-hp", default=None)
    ap.add_argument("--ncu-be", default=None)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    W = bench.build_config(a.config, 0)
    for name, g, base, ncu in (("hp", W["hpg"], 0, a.ncu_hp), ("be", W["beg"], 10000, a.ncu_be)):
        table, rows = PR.build_profiles(g, base, reps=10, ncu_csv=ncu)
        path = os.path.join(a.out, f"{a.config}_{name}.csv")
        PR.write_profile_csv(path, rows)
        tot = sum(r["dur_ns"] for r in rows)
        print(f"== {a.config} {name}: {len(rows)} kernel ops, solo sum {tot / 1e6:.3f} ms -> {path}")
        byfn = collections.defaultdict(lambda: [0, 0])
        for r in rows:
            byfn[r["fn"]][0] += r["dur_ns"]
            byfn[r["fn"]][1] += 1
        for fn, (t, n) in sorted(byfn.items(), key=lambda x: -x[1][0]):
            print(f"   {fn:14s} n={n:4d} {t / 1e6:8.3f} ms {100 * t / tot:5.1f}%")
        for r in sorted(rows, key=lambda r: -r["dur_ns"])[:a.top]:
            bw = r["bytes"] / r["dur_ns"] if r["dur_ns"] else 0
            tf = r["flops"] / r["dur_ns"] / 1e3 if r["dur_ns"] else 0
            print(f"   {r['label']:32s} {r['fn']:12s} {r['cls']} sm={r['sm_needed']:5d} {r['dur_ns'] / 1e3:9.1f} us "
                  f"{bw:7.1f} GB/s {tf:6.2f} TF/s")


if __name__ == "__main__":
    main()
