"""Warm per-launch CUDA-event times of the BE operators at MobileNetV2-b96 shapes (weight-gradient
GEMMs, depthwise fwd / dgrad / wgrad), with algorithmic GB/s. Inputs > L2 for the large shapes.
Also the HP ResNet-50 b4 forward convolutions / 1x1 GEMMs (conv). Usage: python tools/bench_kernels.py [wgs|dw|conv|all]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import _lib as L  # noqa: E402
from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info  # noqa: E402


def timeit(fn, args, reps=20):
    if os.environ.get("BENCH_GRAPH"):   # device-bound: replay a captured graph of `reps` launches
        st = torch.cuda.Stream()
        for _ in range(3):
            orion.kernel_launch(fn, args, st.cuda_stream)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(reps):
                orion.kernel_launch(fn, args, st.cuda_stream)
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps * 1e3
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):
        orion.kernel_launch(fn, args, s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        orion.kernel_launch(fn, args, s)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


def ws(nbytes):
    return torch.zeros(int(nbytes) // 4 + 64, device="cuda")


WGS = [(96, 16, 1204224), (16, 32, 1204224), (24, 96, 301056), (144, 24, 301056), (24, 144, 301056), (32, 144, 75264),
       (192, 32, 75264), (32, 192, 75264), (64, 192, 18816), (384, 64, 18816), (64, 384, 18816), (576, 96, 18816),
       (96, 576, 18816), (160, 576, 4704), (960, 160, 4704), (160, 960, 4704), (320, 960, 4704), (1280, 320, 4704)]
DW = [(96, 112, 32, 1), (96, 112, 96, 2), (96, 56, 144, 1), (96, 56, 144, 2), (96, 28, 192, 1), (96, 28, 192, 2),
      (96, 14, 384, 1), (96, 14, 576, 1), (96, 14, 576, 2), (96, 7, 960, 1)]



HP_CONV = [(4, 56, 56, 64, 64, 3, 1, 1), (4, 56, 56, 128, 128, 3, 2, 1), (4, 28, 28, 128, 128, 3, 1, 1), (4, 28, 28, 256, 256, 3, 2, 1),
           (4, 14, 14, 256, 256, 3, 1, 1), (4, 14, 14, 512, 512, 3, 2, 1), (4, 7, 7, 512, 512, 3, 1, 1),
           (4, 56, 56, 256, 512, 1, 2, 0), (4, 28, 28, 512, 1024, 1, 2, 0), (4, 14, 14, 1024, 2048, 1, 2, 0)]
HP_GEMM = [(12544, 64, 64), (12544, 64, 256), (12544, 256, 64), (12544, 128, 256), (3136, 512, 128), (3136, 128, 512),
           (3136, 256, 512), (784, 1024, 256), (784, 256, 1024), (784, 512, 1024), (196, 2048, 512), (196, 512, 2048)]


def conv():
    tot = 0.0
    for n, h, w_, c, k, r, st, pad in HP_CONV:
        p, q = (h + 2 * pad - r) // st + 1, (w_ + 2 * pad - r) // st + 1
        x, wt, y = torch.randn(n, h, w_, c, device="cuda"), torch.randn(k, r, r, c, device="cuda"), torch.zeros(n, p, q, k, device="cuda")
        wf = ws(L.lib.orion_gemm_workspace_bytes(n * p * q, k, r * r * c))
        a = [x.data_ptr(), wt.data_ptr(), y.data_ptr(), n, h, w_, c, k, r, r, st, pad, p, q, wf.data_ptr(), wf.numel() * 4]
        t = timeit("conv_fwd", a)
        tot += t
        info = kernel_info("conv_fwd", a)
        print(f"conv {n}x{h}x{w_}x{c}->{k} r{r} s{st} {t:7.1f} us {2 * n * p * q * k * r * r * c / t / 1e6:6.1f} TF  grid {info['grid_ctas']} "
              f"{info['kernel'][:40]}")
    for M, N, K in HP_GEMM:
        A, B, C = torch.randn(M, K, device="cuda"), torch.randn(N, K, device="cuda"), torch.zeros(M, N, device="cuda")
        w = ws(L.lib.orion_gemm_workspace_bytes(M, N, K))
        a = [A.data_ptr(), B.data_ptr(), C.data_ptr(), 0, M, N, K, K, K, N, 2, w.data_ptr(), w.numel() * 4]
        t = timeit("gemm", a)
        tot += t
        info = kernel_info("gemm", a)
        print(f"gemm M={M:5d} N={N:5d} K={K:5d} {t:7.1f} us {2 * M * N * K / t / 1e6:6.1f} TF  grid {info['grid_ctas']} {info['kernel'][:40]}")
    print(f"conv+gemm total {tot:.1f} us")


def floor():
    """Graph-replayed duration of trivial launches: the per-kernel floor the HP path pays."""
    x = torch.zeros(1024, device="cuda")
    t = timeit("relu", [x.data_ptr(), x.data_ptr(), x.numel()])
    print(f"relu 1024 floats {t:6.2f} us")
    x = torch.zeros(4 * 56 * 56 * 64, device="cuda")
    t = timeit("relu", [x.data_ptr(), x.data_ptr(), x.numel()])
    print(f"relu 4x56x56x64 {t:6.2f} us")


BE_CWG = [(64, 224, 224, 3, 64, 7, 2, 3), (64, 56, 56, 64, 64, 3, 1, 1), (64, 56, 56, 128, 128, 3, 2, 1), (64, 28, 28, 128, 128, 3, 1, 1), (64, 14, 14, 256, 256, 3, 1, 1),
          (64, 7, 7, 512, 512, 3, 1, 1), (64, 56, 56, 256, 512, 1, 2, 0), (64, 28, 28, 512, 1024, 1, 2, 0)]


def cwg():
    """BE ResNet-50 b64 convolution weight gradients (config 3's dominant BE kernels)."""
    tot = 0.0
    for n, h, w_, c, k, r, st, pad in BE_CWG:
        p, q = (h + 2 * pad - r) // st + 1, (w_ + 2 * pad - r) // st + 1
        x, dy, dw = torch.randn(n, h, w_, c, device="cuda"), torch.randn(n, p, q, k, device="cuda"), torch.zeros(k, r, r, c, device="cuda")
        wf = ws(L.lib.orion_conv_wgrad_workspace_bytes(n, h, w_, c, k, r, r, st, pad))
        a = [x.data_ptr(), dy.data_ptr(), dw.data_ptr(), n, h, w_, c, k, r, r, st, pad, p, q, wf.data_ptr(), wf.numel() * 4]
        t = timeit("conv_wgrad", a)
        tot += t
        info = kernel_info("conv_wgrad", a)
        fl = 2 * n * p * q * k * r * r * c
        print(f"wgrad {n}x{h}x{w_}x{c}->{k} r{r} s{st} {t:8.1f} us {fl / t / 1e6:6.1f} TF ({fl / t / 1e6 / 228:4.2f} of 3xTF32) "
              f"grid {info['grid_ctas']} {info['kernel'][:40]}")
    print(f"conv wgrad total {tot:.1f} us")


BN_SHAPES = [(96 * 112 * 112, 32), (96 * 112 * 112, 96), (96 * 56 * 56, 144), (96 * 56 * 56, 24), (96 * 28 * 28, 192), (96 * 28 * 28, 32),
             (96 * 14 * 14, 384), (96 * 14 * 14, 64), (96 * 14 * 14, 576), (96 * 7 * 7, 960), (96 * 7 * 7, 160), (96 * 7 * 7, 1280)]


def bn():
    """MobileNetV2 b96 BN statistics / backward reduction shapes (rows, C)."""
    tot = 0.0
    for rows, c in BN_SHAPES:
        x, dy = torch.randn(rows, c, device="cuda"), torch.randn(rows, c, device="cuda")
        mean, inv, rm, rv = (torch.zeros(c, device="cuda") for _ in range(4))
        dg, db = torch.zeros(c, device="cuda"), torch.zeros(c, device="cuda")
        w = ws(L.lib.orion_bn_workspace_bytes(rows, c) if hasattr(L.lib, "orion_bn_workspace_bytes") else 64 << 20)
        eps = __import__("struct").unpack("<I", __import__("struct").pack("<f", 1e-5))[0]
        mom = __import__("struct").unpack("<I", __import__("struct").pack("<f", 0.1))[0]
        a1 = [x.data_ptr(), mean.data_ptr(), inv.data_ptr(), rm.data_ptr(), rv.data_ptr(), rows, c, eps, mom, w.data_ptr(), w.numel() * 4]
        a2 = [x.data_ptr(), dy.data_ptr(), mean.data_ptr(), inv.data_ptr(), dg.data_ptr(), db.data_ptr(), rows, c, w.data_ptr(), w.numel() * 4]
        t1, t2 = timeit("bn_stats", a1), timeit("bn_bwd_reduce", a2)
        tot += t1 + t2
        g1 = kernel_info("bn_stats", a1)["grid_ctas"]
        print(f"bn rows={rows:8d} C={c:5d} stats {t1:6.1f} us {4 * rows * c / t1 / 1e3:5.0f} GB/s (grid {g1})  "
              f"bwd_reduce {t2:6.1f} us {8 * rows * c / t2 / 1e3:5.0f} GB/s")
    print(f"bn total {tot:.1f} us")

def stem():
    """MobileNetV2 b96 stem (3x3/2, 3 -> 32 channels): forward and weight gradient."""
    n, h, c, k = 96, 224, 3, 32
    p = 112
    x, wt = torch.randn(n, h, h, c, device="cuda"), torch.randn(k, 3, 3, c, device="cuda")
    y, dy, dw = torch.zeros(n, p, p, k, device="cuda"), torch.randn(n, p, p, k, device="cuda"), torch.zeros(k, 3, 3, c, device="cuda")
    dims = [n, h, h, c, k, 3, 3, 2, 1, p, p]
    wf = ws(max(L.lib.orion_gemm_workspace_bytes(n * p * p, k, 27), L.lib.orion_conv_wgrad_workspace_bytes(n, h, h, c, k, 3, 3, 2, 1)))
    byt = (x.numel() + y.numel()) * 4
    t1 = timeit("conv_fwd", [x.data_ptr(), wt.data_ptr(), y.data_ptr()] + dims + [wf.data_ptr(), wf.numel() * 4])
    t2 = timeit("conv_wgrad", [x.data_ptr(), dy.data_ptr(), dw.data_ptr()] + dims + [wf.data_ptr(), wf.numel() * 4])
    print(f"stem fwd {t1:7.1f} us {byt / t1 / 1e3:5.0f} GB/s   wgrad {t2:7.1f} us {byt / t2 / 1e3:5.0f} GB/s")
    # ResNet-50 HP stem (7x7/2, 3 -> 64) at batch 4
    n, h, k, p = 4, 224, 64, 112
    x, wt, y = torch.randn(n, h, h, 3, device="cuda"), torch.randn(k, 7, 7, 3, device="cuda"), torch.zeros(n, p, p, k, device="cuda")
    dims = [n, h, h, 3, k, 7, 7, 2, 3, p, p]
    wf = ws(L.lib.orion_gemm_workspace_bytes(n * p * p, k, 147))
    a = [x.data_ptr(), wt.data_ptr(), y.data_ptr()] + dims + [wf.data_ptr(), wf.numel() * 4]
    t3 = timeit("conv_fwd", a)
    print(f"resnet stem b4 fwd {t3:7.1f} us {2 * n * p * p * k * 147 / t3 / 1e6:5.1f} TF  {kernel_info('conv_fwd', a)['kernel'][-40:]}")


def attn():
    """Config-4 encoder attention (fp32): B 8, S 192, 8 heads of 64; forward and the two backward ops."""
    B, S, H, d = 8, 192, 8, 64
    D = H * d
    q, k, v, o, do = (torch.randn(B, S, D, device="cuda") for _ in range(5))
    dq, dk, dv = (torch.zeros(B, S, D, device="cuda") for _ in range(3))
    st = torch.zeros(B, H, S, 3, device="cuda")
    t1 = timeit("attention_f32", [q.data_ptr(), k.data_ptr(), v.data_ptr(), o.data_ptr(), B, S, H, d, D, D])
    t2 = timeit("attention_f32_bwd_dq", [q.data_ptr(), k.data_ptr(), v.data_ptr(), do.data_ptr(), dq.data_ptr(), st.data_ptr(), B, S, H, d, D, D])
    t3 = timeit("attention_f32_bwd_dkv", [q.data_ptr(), k.data_ptr(), v.data_ptr(), do.data_ptr(), st.data_ptr(), dk.data_ptr(), dv.data_ptr(),
                                           B, S, H, d, D, D])
    fl = 4 * B * H * S * S * d
    print(f"attn fwd {t1:7.1f} us ({fl / t1 / 1e6:5.1f} TF)  bwd_dq {t2:7.1f} us  bwd_dkv {t3:7.1f} us")


# MobileNetV2 b96 1x1 convolutions: (rows, Cin, Cout); forward y = x W^T (flags 2), data gradient
# dx = dy W (flags 0, B = W [Cout][Cin] MN-major)
G1X1 = [(1204224, 16, 96), (1204224, 32, 16), (301056, 24, 144), (301056, 144, 24), (75264, 32, 192), (75264, 192, 32),
        (18816, 64, 384), (18816, 384, 64)]


def g1x1():
    tot = 0.0
    for M, cin, cout in G1X1:
        x, w, y = torch.randn(M, cin, device="cuda"), torch.randn(cout, cin, device="cuda"), torch.zeros(M, cout, device="cuda")
        dy, dx = torch.randn(M, cout, device="cuda"), torch.zeros(M, cin, device="cuda")
        wf = ws(max(L.lib.orion_gemm_workspace_bytes(M, cout, cin), L.lib.orion_gemm_workspace_bytes(M, cin, cout)))
        af = [x.data_ptr(), w.data_ptr(), y.data_ptr(), 0, M, cout, cin, cin, cin, cout, 2, wf.data_ptr(), wf.numel() * 4]
        ad = [dy.data_ptr(), w.data_ptr(), dx.data_ptr(), 0, M, cin, cout, cout, cin, cin, 0, wf.data_ptr(), wf.numel() * 4]
        t1, t2 = timeit("gemm", af), timeit("gemm", ad)
        tot += t1 + t2
        byt = 4 * M * (cin + cout)
        k1, k2 = kernel_info("gemm", af)["kernel"], kernel_info("gemm", ad)["kernel"]
        print(f"1x1 M={M:8d} {cin:4d}->{cout:4d}  fwd {t1:7.1f} us {byt / t1 / 1e3:5.0f} GB/s  dgrad {t2:7.1f} us {byt / t2 / 1e3:5.0f} GB/s"
              f"  {k1[-30:]} {k2[-30:]}")
    print(f"1x1 total {tot:.1f} us")


def pool():
    """ResNet-50 b64 max-pool 3x3/2 forward and backward (config 3's BE, config 4's HP)."""
    n, h, c, p = 64, 112, 64, 56
    x, y, dy, dx = (torch.randn(n, h, h, c, device="cuda"), torch.zeros(n, p, p, c, device="cuda"), torch.randn(n, p, p, c, device="cuda"),
                    torch.zeros(n, h, h, c, device="cuda"))
    t1 = timeit("maxpool", [x.data_ptr(), y.data_ptr(), n, h, h, c, p, p])
    t2 = timeit("maxpool_bwd", [x.data_ptr(), dy.data_ptr(), dx.data_ptr(), n, h, h, c, p, p])
    print(f"maxpool fwd {t1:7.1f} us {(x.numel() + y.numel()) * 4 / t1 / 1e3:5.0f} GB/s   bwd {t2:7.1f} us "
          f"{(2 * x.numel() + dy.numel()) * 4 / t2 / 1e3:5.0f} GB/s")


def wgs():
    tot = 0.0
    for M, N, K in WGS:
        A, B, C = torch.randn(K, M, device="cuda"), torch.randn(K, N, device="cuda"), torch.zeros(M, N, device="cuda")
        w = ws(L.lib.orion_gemm_workspace_bytes(M, N, K))
        a = [A.data_ptr(), B.data_ptr(), C.data_ptr(), 0, M, N, K, M, N, N, 1, w.data_ptr(), w.numel() * 4]
        t = timeit("gemm", a)
        tot += t
        info = kernel_info("gemm", a)
        print(f"wgrad M={M:5d} N={N:5d} K={K:8d} {t:7.1f} us {4 * K * (M + N) / t / 1e3:6.0f} GB/s "
              f"{2 * M * N * K / t / 1e6:6.1f} TF  grid {info['grid_ctas']} regs {info['regs_per_thread']} {info['kernel'][:40]}")
    print(f"wgrad total {tot:.1f} us")


def dw():
    tot = 0.0
    for n, h, c, st in DW:
        p = (h - 1) // st + 1
        x, dy = torch.randn(n, h, h, c, device="cuda"), torch.randn(n, p, p, c, device="cuda")
        wt = torch.randn(c, 3, 3, 1, device="cuda")
        y, dx, dwt = torch.zeros(n, p, p, c, device="cuda"), torch.zeros(n, h, h, c, device="cuda"), torch.zeros(c, 9, device="cuda")
        dims = [n, h, h, c, c, 3, 3, st, 1, p, p]
        w = ws(L.lib.orion_dw_wgrad_workspace_bytes(n, c, p, p))
        byt = (x.numel() + dy.numel()) * 4
        t1 = timeit("dw_fwd", [x.data_ptr(), wt.data_ptr(), y.data_ptr()] + dims)
        t2 = timeit("dw_dgrad", [dy.data_ptr(), wt.data_ptr(), dx.data_ptr()] + dims)
        t3 = timeit("dw_wgrad", [x.data_ptr(), dy.data_ptr(), dwt.data_ptr()] + dims + [w.data_ptr(), w.numel() * 4])
        tot += t1 + t2 + t3
        print(f"dw n={n} h={h:4d} c={c:4d} s={st}  fwd {t1:7.1f} us {byt / t1 / 1e3:5.0f} GB/s  dgrad {t2:7.1f} us "
              f"{byt / t2 / 1e3:5.0f} GB/s  wgrad {t3:7.1f} us {byt / t3 / 1e3:5.0f} GB/s")
    print(f"dw total {tot:.1f} us")


if __name__ == "__main__":
    torch.cuda.set_device(0)
    what = sys.argv[1] if len(sys.argv) > 1 else "all"
    if what in ("wgs", "all"):
        wgs()
    if what in ("stem", "all"):
        stem()
    if what in ("attn", "all"):
        attn()
    if what in ("g1x1", "all"):
        g1x1()
    if what in ("pool", "all"):
        pool()
    if what in ("dw", "all"):
        dw()
    if what in ("conv", "all"):
        conv()
    if what in ("floor", "all"):
        floor()
    if what in ("cwg", "all"):
        cwg()
    if what in ("bn", "all"):
        bn()
