"""Numerics of the weight-gradient GEMM path as routed in THIS process (env knobs such as
ORION_ATS_MIN_ROWS / ORION_ATC_MIN_AI apply): rel L2 and the elementwise fp32 dot-product bound vs the
fp64 product, determinism, kernel name. Usage: python tools/check_wgrad.py [M N K ...]"""
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import _lib as L  # noqa: E402
from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info  # noqa: E402

CASES = [(96, 16, 1204224), (16, 32, 300037), (24, 96, 100003), (144, 24, 75264), (24, 144, 75271), (32, 144, 75264),
         (192, 32, 75264), (64, 192, 18816), (40, 40, 50000), (100, 36, 65536), (256, 32, 40000)]


def run(M, N, K, seed=5):
    g = torch.Generator().manual_seed(seed)
    A = torch.randn(K, M, generator=g)
    B = torch.randn(K, N, generator=g)
    ref = A.double().t() @ B.double()
    C = torch.zeros(M, N, device="cuda")
    w = torch.zeros(int(L.lib.orion_gemm_workspace_bytes(M, N, K)) // 4 + 64, device="cuda")
    Ad, Bd = A.cuda(), B.cuda()
    args = [Ad.data_ptr(), Bd.data_ptr(), C.data_ptr(), 0, M, N, K, M, N, N, 1, w.data_ptr(), w.numel() * 4]
    kern = kernel_info("gemm", args)["kernel"]
    s = torch.cuda.current_stream().cuda_stream
    orion.kernel_launch("gemm", args, s)
    torch.cuda.synchronize()
    got = C.double().cpu()
    rel = float((got - ref).norm() / ref.norm())
    bound = 4.0 * 2.0 ** -24 * math.sqrt(K) * (A.double().abs().t() @ B.double().abs()) + 1e-30
    worst = float(((got - ref).abs() / bound).max())
    first = C.clone()
    orion.kernel_launch("gemm", args, s)
    torch.cuda.synchronize()
    det = torch.equal(first, C)
    ok = rel < 1e-5 and worst <= 1.0 and det
    print(f"{'OK ' if ok else 'BAD'} M={M} N={N} K={K} rel={rel:.2e} worst={worst:.3f} det={det} {kern[:60]}", flush=True)
    return ok


if __name__ == "__main__":
    torch.cuda.set_device(0)
    a = [int(x) for x in sys.argv[1:]]
    cases = [tuple(a[i:i + 3]) for i in range(0, len(a), 3)] if a else CASES
    bad = sum(not run(*c) for c in cases)
    sys.exit(1 if bad else 0)
