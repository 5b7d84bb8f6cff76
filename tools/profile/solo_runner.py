"""Solo op runner for the offline profiler (§5.2): launches every kernel op of one client's
op list once, in order, directly through the C ABI (no scheduler), so that
`ncu --csv` captures exactly one launch per kernel_id (launch i <-> i-th kernel op)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="rn50_mnv2")
    ap.add_argument("--client", default="be", choices=["hp", "be"])
    ap.add_argument("--only", default=None, help="substring of op labels to launch (others skipped)")
    ap.add_argument("--repeat", type=int, default=1)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    g = bench.build_client(a.config, a.client)
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(a.repeat):
        for fn, args, lab in g.ops:
            if isinstance(fn, str) and (a.only is None or a.only in lab):
                orion.kernel_launch(fn, args, s)
    torch.cuda.synchronize()
    with open(os.path.join(ROOT, "gpurun_out", f"oplist_{a.config}_{a.client}.txt"), "w") as f:
        for i, (fn, args, lab) in enumerate(g.ops):
            if isinstance(fn, str):   # kernels per op launch (2 = split partials + ordered combine)
                f.write(f"{i}\t{fn}\t{lab}\t{kernel_info(fn, args)['launches']}\n")


if __name__ == "__main__":
    main()
