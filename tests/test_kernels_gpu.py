"""Operator parity on the GPU: every liborion kernel, called through the C ABI
(orion_kernel_launch), against the fp64 oracle op (oracle/model.py) on seeded inputs whose shapes
span several tiles plus ragged tails. Tolerance: per-tensor relative L2 <= 1e-5 for single ops
(fp32 storage, fp32 accumulate vs fp64; DESIGN.md §8 derives it), and bitwise determinism
(run twice -> identical bytes)."""
import pytest
import torch

from oracle import model as om
from synth import inputs as si

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_eurosys_stratimk24_b200 as orion
    import paper_conf_eurosys_stratimk24_b200.profiler  # noqa: F401
    from paper_conf_eurosys_stratimk24_b200 import _lib as L


def rel(a, b):
    a = a.detach().double().cpu()
    b = b.detach().double().cpu()
    return float((a - b).norm() / max(float(b.norm()), 1e-30))


def run(fn, args):
    s = torch.cuda.current_stream().cuda_stream
    orion.kernel_launch(fn, [a.data_ptr() if isinstance(a, torch.Tensor) else a for a in args], s)
    torch.cuda.synchronize()


def dev(t):
    return t.cuda().contiguous()


def ws(nbytes):
    return torch.zeros(int(nbytes) // 4 + 64, dtype=torch.float32, device="cuda")


@pytest.mark.parametrize("M,N,K,flags", [(1, 512, 512, 2), (4, 1000, 2048, 2), (3, 37, 129, 2), (32, 512, 512, 2),
                                         (96, 16, 300000, 1), (16, 32, 100000, 1), (196, 2048, 512, 2), (784, 256, 1024, 2),
                                         (256, 256, 256, 0), (300, 200, 520, 1), (130, 70, 300, 2), (257, 129, 333, 3),
                                         (4704, 1280, 320, 2), (1280, 320, 4704, 1), (18816, 96, 576, 2),
                                         (99, 37, 9999, 1), (24, 144, 75264, 1), (128, 32, 300000, 1),
                                         (12544, 16, 96, 0), (20000, 24, 144, 2), (5000, 7, 33, 0), (4097, 32, 512, 2),
                                         (144, 24, 75264, 1), (192, 32, 75264, 1), (32, 192, 75264, 1), (150, 22, 5000, 1),
                                         # multi-tile tcgen05 kernel (>= 296 tiles): ragged M / N / K, unaligned K
                                         (40000, 96, 16, 2), (30000, 144, 20, 0), (20000, 200, 40, 2), (40000, 64, 33, 2),
                                         (301056, 24, 144, 0), (38000, 33, 24, 0), (18816, 384, 64, 2), (4704, 1280, 320, 0),
                                         # skinny A^T B 8x8 register-block variant (ResNet 1x1 weight gradients)
                                         (256, 64, 50000, 1), (64, 256, 50176, 1), (128, 128, 20000, 1), (250, 60, 9999, 1)],
                         ids=lambda v: str(v))
def test_gemm_shapes(M, N, K, flags):
    test_gemm(M, N, K, flags)


@pytest.mark.parametrize("M,N,K,flags", [(1, 512, 512, 2),
                                         (200, 130, 77, 0), (300, 257, 65, 1), (129, 131, 700, 3), (96, 1000, 1280, 2),
                                         (1000, 1280, 96, 1), (64, 96, 20000, 1), (12544, 64, 256, 2)])
def test_gemm(M, N, K, flags):
    A = si.normal((K, M) if flags & 1 else (M, K), 11)
    B = si.normal((N, K) if flags & 2 else (K, N), 12)
    bias = si.normal((N,), 13)
    Ad = A.t() if flags & 1 else A
    Bd = B.t() if flags & 2 else B
    ref = om._r(Ad.double() @ Bd.double() + bias.double())
    C = torch.zeros(M, N, device="cuda")
    w = ws(L.lib.orion_gemm_workspace_bytes(M, N, K))
    args = [dev(A), dev(B), C, dev(bias), M, N, K, A.shape[1], B.shape[1], N, flags, w, w.numel() * 4]
    run("gemm", args)
    assert rel(C, ref) < 1e-5
    first = C.clone()
    run("gemm", args)
    assert torch.equal(first, C), "non-deterministic GEMM"


CONV_CASES = [  # N, H, W, C, K, R, stride, pad
    (2, 17, 15, 3, 32, 3, 2, 1),     # MobileNetV2 stem shape class
    (4, 7, 7, 512, 512, 3, 1, 1),    # ResNet-50 layer4 3x3 at batch 4 (split-K)
    (4, 14, 14, 256, 256, 3, 1, 1),  # layer3 3x3
    (4, 30, 30, 3, 64, 7, 2, 3),     # ResNet stem class
    (2, 14, 14, 64, 70, 3, 1, 1),
    (2, 13, 13, 64, 128, 1, 2, 0),   # 1x1 / stride 2 downsample
    (3, 9, 11, 20, 24, 3, 2, 1),
    (4, 64, 64, 3, 64, 7, 2, 3),     # ResNet stem (direct few-channel wgrad kernel)
    (2, 224, 224, 3, 64, 7, 2, 3),   # ResNet stem at 224 (several tiles per CTA, ragged Q)
    (3, 50, 38, 3, 32, 3, 2, 1),     # MobileNetV2 stem class, ragged
]


@pytest.mark.parametrize("shape", CONV_CASES)
def test_conv_fwd_dgrad_wgrad(shape):
    n, h, w_, c, k, r, st, pad = shape
    x = si.normal((n, h, w_, c), 21)
    wt = si.normal((k, r, r, c), 22) * 0.1
    p, q = (h + 2 * pad - r) // st + 1, (w_ + 2 * pad - r) // st + 1
    dy = si.normal((n, p, q, k), 23)
    dims = [n, h, w_, c, k, r, r, st, pad, p, q]
    y = torch.zeros(n, p, q, k, device="cuda")
    wf = ws(L.lib.orion_gemm_workspace_bytes(n * p * q, k, r * r * c))
    run("conv_fwd", [dev(x), dev(wt), y] + dims + [wf, wf.numel() * 4])
    assert rel(y, om.conv2d_fwd(x, wt, st, pad)) < 1e-5
    dx = torch.zeros(n, h, w_, c, device="cuda")
    wd = ws(L.lib.orion_gemm_workspace_bytes(n * h * w_, c, r * r * k))
    run("conv_dgrad", [dev(dy), dev(wt), dx] + dims + [wd, wd.numel() * 4])
    assert rel(dx, om.conv2d_bwd_data(dy, wt, (n, h, w_, c), st, pad)) < 1e-5
    dw = torch.zeros(k, r, r, c, device="cuda")
    wsb = ws(L.lib.orion_conv_wgrad_workspace_bytes(n, h, w_, c, k, r, r, st, pad))
    run("conv_wgrad", [dev(x), dev(dy), dw] + dims + [wsb, wsb.numel() * 4])
    assert rel(dw, om.conv2d_bwd_weight(x, dy, (k, r, r, c), st, pad)) < 1e-5
    first = dw.clone()
    run("conv_wgrad", [dev(x), dev(dy), dw] + dims + [wsb, wsb.numel() * 4])
    assert torch.equal(first, dw), "non-deterministic conv wgrad"


@pytest.mark.parametrize("n,h,wd,c,st", [(2, 15, 15, 32, 1), (3, 16, 16, 96, 2), (2, 7, 7, 960, 1), (1, 9, 9, 8, 2),
                                          (2, 14, 11, 144, 1), (2, 13, 10, 144, 2), (1, 5, 4, 12, 1), (1, 6, 7, 4, 2),
                                          (3, 28, 28, 192, 2), (1, 1, 1, 16, 1), (1, 2, 3, 8, 2),
                                          # several 16-row bands of the weight-gradient walker, ragged last band
                                          (4, 112, 112, 32, 1), (4, 64, 64, 24, 2), (2, 70, 66, 8, 1), (2, 67, 65, 12, 2)])
def test_depthwise(n, h, wd, c, st):
    """Depthwise 3x3 fwd / dgrad / wgrad (MobileNetV2 shapes incl. C = 144, stride 2, non-square and
    ragged widths that exercise the 3x unrolled window rotation and its remainder)."""
    import parity as PT
    x = si.normal((n, h, wd, c), 31)
    wt = si.normal((c, 3, 3, 1), 32)
    p, q = (h + 2 - 3) // st + 1, (wd + 2 - 3) // st + 1
    dy = si.normal((n, p, q, c), 33)
    dims = [n, h, wd, c, c, 3, 3, st, 1, p, q]
    y = torch.zeros(n, p, q, c, device="cuda")
    run("dw_fwd", [dev(x), dev(wt), y] + dims)
    PT.assert_close("dw_fwd", y, om.conv2d_fwd(x, wt, st, 1, c), 1e-5)
    dx = torch.zeros(n, h, wd, c, device="cuda")
    run("dw_dgrad", [dev(dy), dev(wt), dx] + dims)
    PT.assert_close("dw_dgrad", dx, om.conv2d_bwd_data(dy, wt, (n, h, wd, c), st, 1, c), 1e-5)
    dw = torch.zeros(c, 3, 3, 1, device="cuda")
    wsb = ws(L.lib.orion_dw_wgrad_workspace_bytes(n, c, p, q))
    args = [dev(x), dev(dy), dw] + dims + [wsb, wsb.numel() * 4]
    run("dw_wgrad", args)
    ref = om.conv2d_bwd_weight(x, dy, (c, 3, 3, 1), st, 1, c)
    assert PT.cond_elem(dw, ref, om.conv2d_bwd_weight_abs(x, dy, (c, 3, 3, 1), st, 1, c)) < 1e-5
    assert PT.rel(dw, ref) < 1e-5
    first = dw.clone()
    run("dw_wgrad", args)
    assert torch.equal(first, dw), "non-deterministic depthwise wgrad"


@pytest.mark.parametrize("rows,C", [(4 * 56 * 56, 64), (96 * 7 * 7, 1280), (1000, 24), (12345, 16), (96 * 112 * 112, 32)])
def test_batchnorm(rows, C):
    x = si.normal((rows, C), 41) * 2 + 0.5
    gamma, beta = si.normal((C,), 42), si.normal((C,), 43)
    rm, rv = si.normal((C,), 44) * 0.1, torch.rand(C) + 0.5
    eps = orion.f32bits(1e-5)
    # eval
    y = torch.zeros(rows, C, device="cuda")
    run("bn_eval", [dev(x), y, dev(gamma), dev(beta), dev(rm), dev(rv), rows, C, eps])
    assert rel(y, om.bn_eval(x, gamma, beta, rm, rv)) < 1e-6
    # train stats + apply
    yr, mr, ir, rmr, rvr = om.bn_train_fwd(x, gamma, beta, rm, rv)
    mean, invstd = torch.zeros(C, device="cuda"), torch.zeros(C, device="cuda")
    rmd, rvd = dev(rm), dev(rv)
    wsb = ws(L.lib.orion_bn_workspace_bytes(rows, C))
    run("bn_stats", [dev(x), mean, invstd, rmd, rvd, rows, C, eps, orion.f32bits(0.1), wsb, wsb.numel() * 4])
    assert rel(mean, mr) < 1e-6 and rel(invstd, ir) < 1e-6 and rel(rmd, rmr) < 1e-6 and rel(rvd, rvr) < 1e-6
    run("bn_apply", [dev(x), y, dev(gamma), dev(beta), mean, invstd, rows, C])
    assert rel(y, yr) < 1e-6
    # backward, from the GPU's own saved statistics
    dy = si.normal((rows, C), 45)
    dxr, dgr, dbr = om.bn_bwd(x, dy, gamma, mean.cpu(), invstd.cpu())
    dg, db = torch.zeros(C, device="cuda"), torch.zeros(C, device="cuda")
    run("bn_bwd_reduce", [dev(x), dev(dy), mean, invstd, dg, db, rows, C, wsb, wsb.numel() * 4])
    assert rel(dg, dgr) < 1e-5 and rel(db, dbr) < 1e-5
    dx = torch.zeros(rows, C, device="cuda")
    run("bn_bwd_dx", [dev(x), dev(dy), dx, dev(gamma), mean, invstd, dg, db, rows, C])
    assert rel(dx, dxr) < 1e-5


def test_elementwise_and_pools():
    n = 4 * 56 * 56 * 64 + 3
    x = si.normal((n,), 51) * 4
    dy = si.normal((n,), 52)
    for fn, ref in [("relu", om.relu(x)), ("relu6", om.relu6(x))]:
        y = torch.zeros(n, device="cuda")
        run(fn, [dev(x), y, n])
        assert torch.equal(y.cpu(), ref)
    for fn, ref in [("relu_bwd", om.relu_bwd(x, dy)), ("relu6_bwd", om.relu6_bwd(x, dy)), ("add", om.add(x, dy))]:
        y = torch.zeros(n, device="cuda")
        run(fn, [dev(x), dev(dy), y, n])
        assert torch.equal(y.cpu(), ref), fn
    xm = si.normal((3, 17, 18, 64), 53)
    ym = torch.zeros(3, 9, 9, 64, device="cuda")
    run("maxpool", [dev(xm), ym, 3, 17, 18, 64, 9, 9])
    assert torch.equal(ym.cpu(), om.maxpool3x3s2(xm))
    xa = si.normal((5, 7, 7, 1280), 54)
    ya = torch.zeros(5, 1280, device="cuda")
    run("avgpool", [dev(xa), ya, 5, 49, 1280])
    assert rel(ya, om.avgpool_fwd(xa)) < 1e-6
    dya = si.normal((5, 1280), 55)
    dxa = torch.zeros(5, 7, 7, 1280, device="cuda")
    run("avgpool_bwd", [dev(dya), dxa, 5, 49, 1280])
    assert rel(dxa, om.avgpool_bwd(dya, (5, 7, 7, 1280))) < 1e-6


def test_losses_sgd_colsum():
    z = si.normal((96, 1000), 61) * 3
    lab = si.labels(96, 1000, 62)
    lr, dzr = om.ce_fwd_bwd(z, lab)
    loss, dz = torch.zeros(1, device="cuda"), torch.zeros(96, 1000, device="cuda")
    wsb = ws(L.WS_TICKET_BYTES + 4 * 96)
    run("ce", [dev(z), dev(lab), loss, dz, 96, 1000, wsb, wsb.numel() * 4])
    assert rel(loss, lr) < 1e-6 and rel(dz, dzr) < 1e-5
    y, t = si.normal((32, 512), 63), si.normal((32, 512), 64)
    mr, dyr = om.mse_fwd_bwd(y, t)
    dyy = torch.zeros(32, 512, device="cuda")
    wsb = ws(L.WS_TICKET_BYTES + 8 * 148 * 8)
    run("mse", [dev(y), dev(t), loss, dyy, 32 * 512, wsb, wsb.numel() * 4])
    assert rel(loss, mr) < 1e-6 and rel(dyy, dyr) < 1e-6
    p, gr, v = si.normal((1001,), 65), si.normal((1001,), 66), si.normal((1001,), 67)
    pr, vr = om.sgd(p, gr, v, 0.01, 0.9, False)
    pd, vd = dev(p), dev(v)
    run("sgd", [pd, dev(gr), vd, 1001, orion.f32bits(0.01), orion.f32bits(0.9)])
    assert rel(pd, pr) < 1e-7 and rel(vd, vr) < 1e-7
    A = si.normal((96, 1000), 68)
    out = torch.zeros(1000, device="cuda")
    run("colsum", [dev(A), out, 96, 1000])
    assert rel(out, om._r(A.double().sum(0))) < 1e-6


@pytest.mark.parametrize("M,N", [(1536, 2048), (1536, 512), (1537, 1535), (5, 3), (40000, 37), (32, 512)])
def test_colsum_shapes(M, N):
    """Bias gradients (encoder b8 s192 FFN / projections; ragged rows and columns, N % 4 != 0)."""
    import parity as PT
    A = si.normal((M, N), 69)
    out = torch.zeros(N, device="cuda")
    run("colsum", [dev(A), out, M, N])
    PT.assert_close("colsum", out, om._r(A.double().sum(0)), 1e-6)
    first = out.clone()
    run("colsum", [dev(A), out, M, N])
    assert torch.equal(first, out)


def test_geometry_and_sm_needed():
    """sm_needed = ceil(grid / blocks_per_sm) from the kernel's own launch geometry."""
    A = torch.zeros(4096, 256, device="cuda")
    grid, bps, thr, smem = orion.kernel_geometry("gemm", [A.data_ptr(), A.data_ptr(), A.data_ptr(), 0, 1024, 16, 16, 16, 16, 16, 2, 0, 0])
    assert grid == 1024 // 128 and thr == 320 and bps == 1   # cvf.cu: 128-row tiles, one 16-wide K slab, no split
    # a compute-dense shape routes to a tcgen05 kernel (cvf.cu: 320 threads, ~196 KB dynamic smem)
    grid, bps, thr, smem = orion.kernel_geometry("gemm", [A.data_ptr(), A.data_ptr(), A.data_ptr(), 0, 4096, 256, 256, 256, 256, 256, 0, 0, 0])
    assert thr in (288, 320) and smem > 100_000 and bps == 1
    grid, bps, thr, smem = orion.kernel_geometry("relu", [A.data_ptr(), A.data_ptr(), A.numel()])
    assert grid == min((A.numel() // 4 + 255) // 256, 148 * 8) and 1 <= bps <= 8
    assert orion.profiler.sm_needed("relu", [A.data_ptr(), A.data_ptr(), A.numel()]) == -(-grid // bps)


def test_green_context_partition_runs_and_is_bitwise_equal():
    """A BE client confined to a green-context SM partition (cuGreenCtxCreate, 8-SM granularity)
    produces bitwise the same parameters as on the full GPU (partition-independent kernels)."""
    from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C
    from synth import inputs as si
    P = si.make_params(W.mlp_spec())
    xs = [si.normal((32, 512), si.BE_SEED, sub=i) for i in range(2)]
    g = W.mlp_train_graph(P, xs, xs)
    be = C.BEClient(g)
    C.run_session(be=be, be_iters=6)
    ref = g.params.flat.cpu().clone()
    g.params.reset()
    C.run_session(be=be, be_iters=6, be_partition_sms=16)
    assert torch.equal(g.params.flat.cpu(), ref)
