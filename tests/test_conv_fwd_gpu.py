"""Forward convolutions and dense B^T GEMMs on the TMA-im2col tcgen05 kernel (csrc/kernels/cvf.cu):
the convolutions of the HP ResNet inference and the BE ResNet training step, against the
fp64 oracle (oracle/model.py conv2d_fwd / linear_fwd).

Checks per case:
  * the cvf kernel really ran (orion_kernel_info names cvf_kernel) -- with the thread-block cluster
    split where the plan uses one;
  * per-tensor relative L2 <= 1e-5 (single fp32 op);
  * elementwise |y - ref| <= 4 u sqrt(K) (|x| * |w|) + u |ref|: the rounding bound of each output's
    length-K fp32 dot product (K = R S C) plus the oracle's own rounding to fp32 -- it catches a
    wrong tap, a shifted box or a ragged tail that a per-tensor norm would average away;
  * a second launch reproduces the bytes (fixed summation order, also across the cluster)."""
import math

import pytest
import torch

from oracle import model as om
from synth import inputs as si

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_eurosys_stratimk24_b200 as orion
    from paper_conf_eurosys_stratimk24_b200 import _lib as L
    from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info

U = 2.0 ** -24


def _launch(fn, args):
    s = torch.cuda.current_stream().cuda_stream
    orion.kernel_launch(fn, args, s)
    torch.cuda.synchronize()


def _check(got, ref, absref, K):
    g, r, a = got.double().cpu(), ref.double(), absref.double()
    rel = float((g - r).norm() / r.norm())
    assert rel < 1e-5, rel
    bound = 4 * U * math.sqrt(K) * a + U * r.abs() + 1e-30
    worst = float(((g - r).abs() / bound).max())
    assert worst <= 1.0, f"elementwise error {worst:.3f} x the fp32 dot-product bound"


CONV = [  # N, H, W, C, K, R, stride, pad
    (4, 56, 56, 64, 64, 3, 1, 1),      # HP ResNet-50 b4 layer1 3x3 (112-row tiles, cluster split)
    (4, 56, 56, 128, 128, 3, 2, 1),    # layer2.0 conv2 stride 2 (v1.5)
    (4, 28, 28, 128, 128, 3, 1, 1),    # layer2 3x3
    (4, 14, 14, 256, 256, 3, 1, 1),    # layer3 3x3 (balanced 7-row blocks)
    (4, 7, 7, 512, 512, 3, 1, 1),      # layer4 3x3 (two images per tile, 8-CTA cluster)
    (4, 56, 56, 256, 512, 1, 2, 0),    # layer2.0 downsample 1x1 stride 2
    (4, 14, 14, 1024, 2048, 1, 2, 0),  # layer4.0 downsample
    (8, 56, 56, 64, 64, 3, 1, 1),      # BE-size tile grid (split 1, several waves)
    (3, 9, 11, 36, 40, 3, 2, 1),       # ragged everything, C % 32 != 0 (zero-filled channel block)
    (2, 5, 150, 20, 68, 3, 1, 1),      # Q > 128: column blocks
    (1, 12, 12, 8, 24, 5, 1, 2),       # 5x5, C = 8
]


@pytest.mark.parametrize("n,h,w,c,k,r,st,pad", CONV, ids=lambda v: str(v))
def test_conv_fwd_tensor_path(n, h, w, c, k, r, st, pad):
    x = si.normal((n, h, w, c), 51)
    wt = si.normal((k, r, r, c), 52) * 0.1
    p, q = (h + 2 * pad - r) // st + 1, (w + 2 * pad - r) // st + 1
    y = torch.full((n, p, q, k), float("nan"), device="cuda")
    xd, wd = x.cuda(), wt.cuda()
    args = [xd.data_ptr(), wd.data_ptr(), y.data_ptr(), n, h, w, c, k, r, r, st, pad, p, q, 0, 0]
    assert "cvf_kernel" in kernel_info("conv_fwd", args)["kernel"]
    _launch("conv_fwd", args)
    _check(y, om.conv2d_fwd(x, wt, st, pad), om.conv2d_fwd(x.abs(), wt.abs(), st, pad), r * r * c)
    first = y.clone()
    _launch("conv_fwd", args)
    assert torch.equal(first, y), "non-deterministic convolution"


GEMM = [  # M, N, K, bias: y = x W^T (+ b), the 1x1 convolutions / Linear layers routed to cvf
    (3136, 64, 256, False),    # HP layer1 conv1
    (784, 512, 1024, False),   # HP layer4.0 conv1 class
    (196, 2048, 512, False),   # layer4 conv3
    (1000, 100, 36, True),     # ragged K (zero-filled block), ragged N, bias
    (129, 200, 64, True),
]


@pytest.mark.parametrize("M,N,K,bias", GEMM, ids=lambda v: str(v))
def test_gemm_bt_tensor_path(M, N, K, bias):
    A = si.normal((M, K), 61)
    W = si.normal((N, K), 62) * 0.1
    b = si.normal((N,), 63) if bias else None
    C = torch.full((M, N), float("nan"), device="cuda")
    Ad, Wd = A.cuda(), W.cuda()
    bd = b.cuda() if bias else None
    nws = L.lib.orion_gemm_workspace_bytes(M, N, K)
    w = torch.zeros(int(nws) // 4 + 64, device="cuda")
    args = [Ad.data_ptr(), Wd.data_ptr(), C.data_ptr(), bd.data_ptr() if bias else 0, M, N, K, K, K, N, 2, w.data_ptr(), w.numel() * 4]
    kern = kernel_info("gemm", args)["kernel"]
    _launch("gemm", args)
    ref = om.linear_fwd(A, W, b)
    absref = om.linear_fwd(A.abs(), W.abs(), b.abs() if bias else None)
    _check(C, ref, absref, K + 1)
    if M * N >= 128 * 64 and M > 8:
        assert "cvf_kernel" in kern or "tmk" in kern or "tcm" in kern or "rows" in kern, kern
    first = C.clone()
    _launch("gemm", args)
    assert torch.equal(first, C)


GEMM_NN = [  # M, N, K: C = A B with B given [K][N] (flags = 0): 1x1-conv / Linear data gradients
    (4704, 160, 960),    # MobileNetV2 b96 features.16 expand data gradient (7x7 maps)
    (4704, 960, 320),    # features.18 data gradient
    (784, 1024, 512),
    (1000, 100, 36),     # ragged K / N
    (129, 200, 64),
]


@pytest.mark.parametrize("M,N,K", GEMM_NN, ids=lambda v: str(v))
def test_gemm_nn_tensor_path(M, N, K):
    """MN-major B straight from TMA (128-byte swizzle with 32-byte atoms) into the transposed-B MMA."""
    A = si.normal((M, K), 71)
    B = si.normal((K, N), 72) * 0.1
    C = torch.full((M, N), float("nan"), device="cuda")
    Ad, Bd = A.cuda(), B.cuda()
    nws = L.lib.orion_gemm_workspace_bytes(M, N, K)
    w = torch.zeros(int(nws) // 4 + 64, device="cuda")
    args = [Ad.data_ptr(), Bd.data_ptr(), C.data_ptr(), 0, M, N, K, K, N, N, 0, w.data_ptr(), w.numel() * 4]
    kern = kernel_info("gemm", args)["kernel"]
    _launch("gemm", args)
    ref = om.linear_fwd(A, B.t().contiguous(), None)
    absref = om.linear_fwd(A.abs(), B.abs().t().contiguous(), None)
    _check(C, ref, absref, K)
    assert "cvf_kernel" in kern or "tmk" in kern, kern   # streaming shapes (>= 296 tiles) keep the multi-tile kernel
    first = C.clone()
    _launch("gemm", args)
    assert torch.equal(first, C)
