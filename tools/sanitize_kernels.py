"""One small launch of every kernel family, for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): the tcgen05 + TMA + mbarrier GEMMs (tc, tcm, tmk, bf16), the TMA-fed streaming weight
gradient (wgs), depthwise, BN and the elementwise kernels. Shapes are small so racecheck finishes."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import _lib as L  # noqa: E402
from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info  # noqa: E402


def ws(n):
    return torch.zeros(int(n) // 4 + 64, device="cuda")


def gemm(M, N, K, flags, bias=False):
    A = torch.randn((K, M) if flags & 1 else (M, K), device="cuda")
    B = torch.randn((N, K) if flags & 2 else (K, N), device="cuda")
    C = torch.zeros(M, N, device="cuda")
    b = torch.randn(N, device="cuda") if bias else None
    w = ws(L.lib.orion_gemm_workspace_bytes(M, N, K))
    a = [A.data_ptr(), B.data_ptr(), C.data_ptr(), b.data_ptr() if bias else 0, M, N, K, A.shape[1], B.shape[1], N, flags,
         w.data_ptr(), w.numel() * 4]
    print("gemm", M, N, K, flags, kernel_info("gemm", a)["kernel"][:60], flush=True)
    orion.kernel_launch("gemm", a, torch.cuda.current_stream().cuda_stream)


def main():
    torch.cuda.set_device(0)
    s = torch.cuda.current_stream().cuda_stream
    gemm(300, 200, 520, 0)          # tcgen05 tiled (cp.async producers, split-K)
    gemm(20000, 96, 16, 2, True)    # tmk: TMA-fed multi-tile tcgen05
    gemm(40000, 64, 33, 2)          # tcm
    gemm(96, 16, 30000, 1)          # wgs (TMA ring, mbarriers, split combine)
    gemm(160, 960, 600, 1)          # wgs, many tiles
    gemm(4096, 32, 512, 2)          # rows kernel
    x = torch.randn(256, 768, device="cuda").to(torch.bfloat16)
    wb = torch.randn(3072, 768, device="cuda").to(torch.bfloat16)
    y = torch.zeros(256, 3072, device="cuda", dtype=torch.bfloat16)
    orion.kernel_launch("gemm_bf16", [x.data_ptr(), wb.data_ptr(), y.data_ptr(), 0, 256, 3072, 768], s)
    print("gemm_bf16", flush=True)
    n, h, c = 2, 14, 144
    xx, wt = torch.randn(n, h, h, c, device="cuda"), torch.randn(c, 3, 3, 1, device="cuda")
    for st in (1, 2):
        p = (h - 1) // st + 1
        dy, yy, dx, dw = (torch.randn(n, p, p, c, device="cuda"), torch.zeros(n, p, p, c, device="cuda"),
                          torch.zeros(n, h, h, c, device="cuda"), torch.zeros(c, 9, device="cuda"))
        dims = [n, h, h, c, c, 3, 3, st, 1, p, p]
        w = ws(L.lib.orion_dw_wgrad_workspace_bytes(n, c, p, p))
        orion.kernel_launch("dw_fwd", [xx.data_ptr(), wt.data_ptr(), yy.data_ptr()] + dims, s)
        orion.kernel_launch("dw_dgrad", [dy.data_ptr(), wt.data_ptr(), dx.data_ptr()] + dims, s)
        orion.kernel_launch("dw_wgrad", [xx.data_ptr(), dy.data_ptr(), dw.data_ptr()] + dims + [w.data_ptr(), w.numel() * 4], s)
    print("depthwise", flush=True)
    rows, C = 5000, 96
    xb, dyb = torch.randn(rows, C, device="cuda"), torch.randn(rows, C, device="cuda")
    v = [torch.zeros(C, device="cuda") for _ in range(6)]
    w = ws(L.lib.orion_bn_workspace_bytes(rows, C))
    orion.kernel_launch("bn_stats", [xb.data_ptr(), v[0].data_ptr(), v[1].data_ptr(), v[2].data_ptr(), v[3].data_ptr(), rows, C,
                                     orion.f32bits(1e-5), orion.f32bits(0.1), w.data_ptr(), w.numel() * 4], s)
    orion.kernel_launch("bn_bwd_reduce", [xb.data_ptr(), dyb.data_ptr(), v[0].data_ptr(), v[1].data_ptr(), v[4].data_ptr(),
                                          v[5].data_ptr(), rows, C, w.data_ptr(), w.numel() * 4], s)
    out = torch.zeros(C, device="cuda")
    orion.kernel_launch("colsum", [xb.data_ptr(), out.data_ptr(), rows, C], s)
    print("bn / colsum", flush=True)
    torch.cuda.synchronize()
    print("done", flush=True)


if __name__ == "__main__":
    main()
