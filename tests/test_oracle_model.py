"""Pins for the model oracle (oracle/model.py) — each against something other than itself:
explicit-loop definitions on tiny shapes, adjoint identities and central finite differences for
backward ops, closed forms, and TorchVision's own model definitions (the models the paper ran,
PAPER.md P:955-958) evaluated in fp64 with autograd."""
import math

import pytest
import torch

from oracle import model as om
from synth import inputs as si

torch.manual_seed(0)
D = torch.float64


def _rand(*shape, seed=0):
    g = torch.Generator().manual_seed(seed)
    return torch.randn(*shape, generator=g, dtype=torch.float32)


def conv_loops(x, w, stride, pad, groups):
    n, h, wd, c = x.shape
    o, kh, kw, ig = w.shape
    ho, wo = (h + 2 * pad - kh) // stride + 1, (wd + 2 * pad - kw) // stride + 1
    og = o // groups
    y = torch.zeros(n, ho, wo, o, dtype=D)
    for b in range(n):
        for i in range(ho):
            for j in range(wo):
                for oc in range(o):
                    gi = oc // og
                    acc = 0.0
                    for u in range(kh):
                        for v in range(kw):
                            hi, wi = i * stride - pad + u, j * stride - pad + v
                            if 0 <= hi < h and 0 <= wi < wd:
                                for ci in range(ig):
                                    acc += float(x[b, hi, wi, gi * ig + ci]) * float(w[oc, u, v, ci])
                    y[b, i, j, oc] = acc
    return y


@pytest.mark.parametrize("stride,pad,k,groups,cin,cout", [(1, 0, 1, 1, 3, 4), (2, 1, 3, 1, 2, 3), (2, 3, 7, 1, 3, 2),
                                                           (1, 1, 3, 4, 4, 4), (2, 1, 3, 3, 3, 3)])
def test_conv_fwd_loops(stride, pad, k, groups, cin, cout):
    x = _rand(2, 7, 6, cin, seed=1)
    w = _rand(cout, k, k, cin // groups, seed=2)
    y = om.conv2d_fwd(x, w, stride, pad, groups)
    ref = conv_loops(x, w, stride, pad, groups)
    assert y.dtype == torch.float32
    torch.testing.assert_close(y.double(), ref, rtol=1e-6, atol=1e-6)


@pytest.mark.parametrize("stride,pad,k,groups,cin,cout", [(1, 0, 1, 1, 3, 4), (2, 1, 3, 1, 2, 3), (1, 1, 3, 4, 4, 4),
                                                           (2, 1, 3, 6, 6, 6)])
def test_conv_bwd_adjoint(stride, pad, k, groups, cin, cout):
    """<conv(x,w), dy> = <x, dgrad(dy,w)> = <w, wgrad(x,dy)> (bilinearity; catches transposes)."""
    x = _rand(2, 9, 8, cin, seed=3)
    w = _rand(cout, k, k, cin // groups, seed=4)
    ref = torch.from_numpy(conv_loops(x, w, stride, pad, groups).numpy())
    dy = _rand(*ref.shape, seed=5)
    lhs = (ref * dy.double()).sum()
    dx = om.conv2d_bwd_data(dy, w, tuple(x.shape), stride, pad, groups)
    dw = om.conv2d_bwd_weight(x, dy, tuple(w.shape), stride, pad, groups)
    assert abs(float((x.double() * dx.double()).sum() - lhs)) < 1e-5 * (1 + abs(float(lhs)))
    assert abs(float((w.double() * dw.double()).sum() - lhs)) < 1e-5 * (1 + abs(float(lhs)))
    # and element-wise dw against loops: dw[o,u,v,i] = sum x[..] dy[..]
    n, h, wd, _ = x.shape
    ho, wo = dy.shape[1], dy.shape[2]
    og = cout // groups
    for oc in range(0, cout, max(1, cout // 2)):
        for ci in range(cin // groups):
            acc = 0.0
            for b in range(n):
                for i in range(ho):
                    for j in range(wo):
                        hi, wi = i * stride - pad, j * stride - pad      # tap (u, v) = (0, 0)
                        if 0 <= hi < h and 0 <= wi < wd:
                            acc += float(x[b, hi, wi, (oc // og) * (cin // groups) + ci]) * float(dy[b, i, j, oc])
            assert abs(float(dw[oc, 0, 0, ci]) - acc) < 1e-4 * (1 + abs(acc))


def _fd_check(f, x, eps=1e-6, n=6, seed=0):
    """Central finite differences of scalar f at a few random coordinates of x (fp64)."""
    g = torch.Generator().manual_seed(seed)
    idx = torch.randint(0, x.numel(), (n,), generator=g)
    out = []
    for i in idx:
        xp = x.clone().reshape(-1); xp[i] += eps
        xm = x.clone().reshape(-1); xm[i] -= eps
        out.append((int(i), (f(xp.reshape(x.shape)) - f(xm.reshape(x.shape))) / (2 * eps)))
    return out


@pytest.fixture
def exact(monkeypatch):
    """Run the oracle without the fp32 storage rounding so finite differences are exact-ish."""
    monkeypatch.setattr(om, "_r", lambda t: t)
    return om


def test_linear_and_bwd(exact):
    x = _rand(3, 5, seed=1).double(); w = _rand(4, 5, seed=2).double(); b = _rand(4, seed=3).double()
    y = exact.linear_fwd(x, w, b)
    for i in range(3):
        for o in range(4):
            assert abs(float(y[i, o]) - (sum(float(x[i, k]) * float(w[o, k]) for k in range(5)) + float(b[o]))) < 1e-12
    r = _rand(3, 4, seed=4).double()
    dx, dw, db = exact.linear_bwd(x, w, r)
    for i, v in _fd_check(lambda xx: float((exact.linear_fwd(xx, w, b) * r).sum()), x):
        assert abs(float(dx.reshape(-1)[i]) - v) < 1e-6
    for i, v in _fd_check(lambda ww: float((exact.linear_fwd(x, ww, b) * r).sum()), w):
        assert abs(float(dw.reshape(-1)[i]) - v) < 1e-6
    for i, v in _fd_check(lambda bb: float((exact.linear_fwd(x, w, bb) * r).sum()), b, n=4):
        assert abs(float(db.reshape(-1)[i]) - v) < 1e-6


def test_bn_train_closed_form_and_fd(exact):
    x = (_rand(4, 3, 3, 5, seed=1) * 3 + 1).double()
    gamma = _rand(5, seed=2).double(); beta = _rand(5, seed=3).double()
    rm = torch.zeros(5, dtype=D); rv = torch.ones(5, dtype=D)
    y, mean, invstd, rm2, rv2 = exact.bn_train_fwd(x, gamma, beta, rm, rv)
    flat = y.reshape(-1, 5)
    # closed form: normalised output has per-channel mean beta and (biased) std |gamma|*sqrt(var/(var+eps))
    torch.testing.assert_close(flat.mean(0), beta, rtol=0, atol=1e-10)
    var = x.reshape(-1, 5).var(0, unbiased=False)
    torch.testing.assert_close(flat.std(0, unbiased=False), gamma.abs() * torch.sqrt(var / (var + 1e-5)), rtol=1e-10, atol=1e-10)
    # running stats: momentum 0.1 with the unbiased variance (torch semantics)
    torch.testing.assert_close(rm2, 0.1 * x.reshape(-1, 5).mean(0))
    torch.testing.assert_close(rv2, 0.9 + 0.1 * x.reshape(-1, 5).var(0, unbiased=True))
    r = _rand(4, 3, 3, 5, seed=9).double()
    dx, dg, db = exact.bn_bwd(x, r, gamma, mean, invstd)
    f = lambda xx: float((exact.bn_train_fwd(xx, gamma, beta, rm, rv)[0] * r).sum())
    for i, v in _fd_check(f, x, eps=1e-5):
        assert abs(float(dx.reshape(-1)[i]) - v) < 1e-6 * (1 + abs(v))
    fg = lambda gg: float((exact.bn_train_fwd(x, gg, beta, rm, rv)[0] * r).sum())
    for i, v in _fd_check(fg, gamma, n=3):
        assert abs(float(dg[i]) - v) < 1e-6 * (1 + abs(v))
    torch.testing.assert_close(db, r.reshape(-1, 5).sum(0))


def test_bn_eval_special_case():
    """rm=0, rv=1-eps, gamma=1, beta=0 -> identity."""
    x = _rand(2, 2, 2, 3)
    y = om.bn_eval(x, torch.ones(3), torch.zeros(3), torch.zeros(3), torch.full((3,), 1 - 1e-5, dtype=torch.float64))
    torch.testing.assert_close(y, x, rtol=1e-6, atol=1e-7)


def test_relu_family():
    x = torch.tensor([-1.0, 0.0, 0.5, 6.0, 7.0])
    dy = torch.ones(5)
    assert om.relu(x).tolist() == [0, 0, 0.5, 6, 7]
    assert om.relu_bwd(x, dy).tolist() == [0, 0, 1, 1, 1]
    assert om.relu6(x).tolist() == [0, 0, 0.5, 6, 6]
    assert om.relu6_bwd(x, dy).tolist() == [0, 0, 1, 0, 0]


def test_maxpool_loops():
    x = _rand(2, 7, 8, 3, seed=5)
    y = om.maxpool3x3s2(x)
    assert y.shape == (2, 4, 4, 3)
    for b in range(2):
        for i in range(4):
            for j in range(4):
                for c in range(3):
                    m = -math.inf
                    for u in range(3):
                        for v in range(3):
                            hi, wi = 2 * i - 1 + u, 2 * j - 1 + v
                            if 0 <= hi < 7 and 0 <= wi < 8:
                                m = max(m, float(x[b, hi, wi, c]))
                    assert float(y[b, i, j, c]) == m


def test_avgpool_and_bwd(exact):
    x = _rand(2, 3, 4, 5, seed=6).double()
    y = exact.avgpool_fwd(x)
    torch.testing.assert_close(y[1, 2], x[1, :, :, 2].sum() / 12)
    r = _rand(2, 5, seed=7).double()
    dx = exact.avgpool_bwd(r, tuple(x.shape))
    for i, v in _fd_check(lambda xx: float((exact.avgpool_fwd(xx) * r).sum()), x):
        assert abs(float(dx.reshape(-1)[i]) - v) < 1e-8


def test_ce_closed_form_and_fd(exact):
    z = torch.zeros(3, 10, dtype=D)
    loss, dz = exact.ce_fwd_bwd(z, torch.tensor([1, 2, 3]))
    assert abs(float(loss) - math.log(10)) < 1e-12
    torch.testing.assert_close(dz.sum(1), torch.zeros(3, dtype=D), atol=1e-15, rtol=0)
    z = _rand(4, 7, seed=8).double() * 3
    lab = torch.tensor([0, 6, 3, 3])
    loss, dz = exact.ce_fwd_bwd(z, lab)
    for i, v in _fd_check(lambda zz: float(exact.ce_fwd_bwd(zz, lab)[0]), z):
        assert abs(float(dz.reshape(-1)[i]) - v) < 1e-8


def test_mse_closed_form(exact):
    y = torch.tensor([[1.0, 2.0], [3.0, 5.0]], dtype=D)
    t = torch.tensor([[0.0, 2.0], [3.0, 1.0]], dtype=D)
    loss, dy = exact.mse_fwd_bwd(y, t)
    assert float(loss) == (1 + 0 + 0 + 16) / 4
    assert dy.tolist() == [[0.5, 0.0], [0.0, 2.0]]


def test_sgd_sequence():
    p = torch.tensor([1.0]); g1 = torch.tensor([0.5]); g2 = torch.tensor([0.25])
    p1, v1 = om.sgd(p, g1, None, 0.1, 0.9, True)        # v = g; p = 1 - 0.05
    assert abs(float(p1) - 0.95) < 1e-7 and float(v1) == 0.5
    p2, v2 = om.sgd(p1, g2, v1, 0.1, 0.9, False)         # v = 0.45 + 0.25 = 0.7; p = 0.95 - 0.07
    assert abs(float(v2) - 0.7) < 1e-7 and abs(float(p2) - 0.88) < 1e-7
    p3, _ = om.sgd(p, g1, None, 0.1, 0.0, True)
    assert abs(float(p3) - 0.95) < 1e-7


def test_mlp_train_step_vs_autograd():
    spec = om.mlp_spec(64)
    P = si.make_params(spec)
    x = si.normal((8, 64), 2); t = si.normal((8, 64), 2, sub=1)
    loss, newP, grads = om.mlp_train_step(P, x, t, lr=0.01)
    Pd = {k: v.double().requires_grad_() for k, v in P.items()}
    h = x.double()
    for i in range(3):
        h = h @ Pd[f"fc{i}.w"].t() + Pd[f"fc{i}.b"]
        if i < 2:
            h = torch.relu(h)
    L = ((h - t.double()) ** 2).mean()
    L.backward()
    assert abs(float(loss) - float(L)) < 1e-6 * float(L)
    for k in P:
        ref = Pd[k].grad
        assert float((grads[k].double() - ref).norm() / ref.norm()) < 1e-5, k
        torch.testing.assert_close(newP[k].double(), (P[k].double() - 0.01 * ref), rtol=1e-6, atol=1e-7)


def _to_tv(P, tv_model, rename):
    """Load oracle params (OHWI convs) into a torchvision module (OIHW), fp64."""
    sd = tv_model.state_dict()
    for k, v in P.items():
        tk = rename(k)
        t = v.double()
        if t.dim() == 4:
            t = t.permute(0, 3, 1, 2)
        assert sd[tk].shape == t.shape, (k, tk, sd[tk].shape, t.shape)
        sd[tk] = t
    tv_model.load_state_dict(sd)


def _rn_rename(k):
    k = k.replace(".gamma", ".weight").replace(".beta", ".bias").replace(".rmean", ".running_mean").replace(".rvar", ".running_var")
    k = k.replace(".down.w", ".downsample.0.weight").replace(".downbn.", ".downsample.1.")
    k = k.replace(".w", ".weight").replace(".b", ".bias") if k.endswith((".w", ".b")) else k
    return k


def test_resnet50_infer_vs_torchvision():
    tv = pytest.importorskip("torchvision")
    spec = om.resnet_spec()
    P = si.make_params(spec)
    m = tv.models.resnet50().double().eval()
    _to_tv(P, m, _rn_rename)
    x = si.normal((1, 64, 64, 3), 1)
    y = om.resnet_infer(P, x)
    with torch.no_grad():
        ref = m(x.double().permute(0, 3, 1, 2))
    assert float((y.double() - ref).norm() / ref.norm()) < 1e-5


def _mn_rename(k):
    # features.0 stem; block internals; features.18; classifier
    import re
    k = k.replace(".gamma", ".weight").replace(".beta", ".bias").replace(".rmean", ".running_mean").replace(".rvar", ".running_var")
    if k.startswith("features.0."):
        return k.replace("features.0.w", "features.0.0.weight").replace("features.0.bn.", "features.0.1.")
    if k.startswith("features.18."):
        return k.replace("features.18.w", "features.18.0.weight").replace("features.18.bn.", "features.18.1.")
    if k.startswith("classifier."):
        return k.replace("classifier.w", "classifier.1.weight").replace("classifier.b", "classifier.1.bias")
    mobj = re.match(r"features\.(\d+)\.(\w+?)(_bn)?\.(\w+)$", k)
    i, part, bn, leaf = int(mobj.group(1)), mobj.group(2), mobj.group(3), mobj.group(4)
    expand = om.mnv2_blocks()[i - 1][5]
    idx = {"expand": 0, "dw": 1 if expand else 0, "project": 2 if expand else 1}[part]
    if part == "project":
        base = f"features.{i}.conv.{idx if not bn else idx + 1}"
        return base + (".weight" if leaf == "w" else f".{leaf}")
    sub = 1 if bn else 0
    return f"features.{i}.conv.{idx}.{sub}" + (".weight" if leaf == "w" else f".{leaf}")


def test_mnv2_train_step_vs_torchvision():
    """Tiny MobileNetV2 (32x32 input, batch 4, 10 classes): loss, every gradient, BN running
    stats and the SGD(momentum) update against torchvision's model + fp64 autograd."""
    tv = pytest.importorskip("torchvision")
    spec = om.mnv2_spec(num_classes=10)
    P = si.make_params(spec)
    m = tv.models.mobilenet_v2(num_classes=10).double().train()
    m.classifier[0].p = 0.0
    _to_tv(P, m, _mn_rename)
    x = si.normal((4, 64, 64, 3), 2)
    lab = si.labels(4, 10, 2)
    loss, newP, newV, g = om.mnv2_train_step(P, {}, x, lab, first=True)
    out = m(x.double().permute(0, 3, 1, 2))
    L = torch.nn.functional.cross_entropy(out, lab.long())
    L.backward()
    assert abs(float(loss) - float(L)) < 1e-5 * float(L)
    named = dict(m.named_parameters())
    bufs = dict(m.named_buffers())
    worst = 0.0
    for k in g:
        ref = named[_mn_rename(k)].grad
        if ref.dim() == 4:
            ref = ref.permute(0, 2, 3, 1)
        # beta of a BN feeding conv -> train-mode BN has an exactly-zero true gradient (the next
        # BN removes per-channel shifts); compare against an absolute floor there.
        err = float((g[k].double() - ref).norm() / max(float(ref.norm()), 1e-3))
        worst = max(worst, err)
        assert err < 1e-3, (k, err)
    for k in P:
        if k.endswith((".rmean", ".rvar")):
            torch.testing.assert_close(newP[k].double(), bufs[_mn_rename(k)], rtol=1e-5, atol=1e-6)
    k = "classifier.w"
    torch.testing.assert_close(newP[k].double(), P[k].double() - 0.01 * named[_mn_rename(k)].grad, rtol=1e-5, atol=1e-7)
    assert worst < 1e-3


def test_abs_sum_scales():
    """The error-model scales (trace["abs"]) are absolute-term sums: they bound |gradient|
    elementwise (triangle inequality) and equal it when every term has one sign."""
    g = torch.Generator().manual_seed(5)
    x = torch.randn(2, 5, 6, 4, generator=g, dtype=torch.float32)
    dy = torch.randn(2, 5, 6, 3, generator=g, dtype=torch.float32)
    w_shape = (3, 1, 1, 4)
    dw = om.conv2d_bwd_weight(x, dy, w_shape).double()
    A = om.conv2d_bwd_weight_abs(x, dy, w_shape)
    assert bool((A >= dw.abs() - 1e-6).all())
    assert torch.allclose(om.conv2d_bwd_weight_abs(x.abs(), dy.abs(), w_shape), om.conv2d_bwd_weight(x.abs(), dy.abs(), w_shape).double(), rtol=1e-6)
    dw3 = om.conv2d_bwd_weight(x, torch.randn(2, 5, 6, 4, generator=g), (4, 3, 3, 1), 1, 1, groups=4)
    assert om.conv2d_bwd_weight_abs(x, torch.randn(2, 5, 6, 4, generator=g), (4, 3, 3, 1), 1, 1, groups=4).shape == dw3.shape
    z = torch.randn(2, 5, 6, 4, generator=g, dtype=torch.float32)
    dyb = torch.randn(2, 5, 6, 4, generator=g, dtype=torch.float32)
    mean, invstd = z.double().reshape(-1, 4).mean(0).float(), (1 / z.double().reshape(-1, 4).std(0, unbiased=False)).float()
    _, dgam, dbet = om.bn_bwd(z, dyb, torch.ones(4), mean, invstd)
    Ag, Ab = om.bn_bwd_abs(z, dyb, mean, invstd)
    assert bool((Ag >= dgam.double().abs() - 1e-6).all()) and bool((Ab >= dbet.double().abs() - 1e-6).all())
    assert torch.allclose(om.bn_bwd_abs(z, dyb.abs(), mean, invstd)[1], om.bn_bwd(z, dyb.abs(), torch.ones(4), mean, invstd)[2].double(), rtol=1e-6)


def test_mnv2_infer_vs_torchvision():
    """Inf-inf BE client: MobileNetV2 inference with seeded eval statistics vs torchvision, fp64."""
    tv = pytest.importorskip("torchvision")
    P = si.make_params(om.mnv2_spec(num_classes=10, eval_stats=True))
    m = tv.models.mobilenet_v2(num_classes=10).double().eval()
    _to_tv(P, m, _mn_rename)
    x = si.normal((2, 64, 64, 3), 3)
    y = om.mnv2_infer(P, x)
    with torch.no_grad():
        ref = m(x.double().permute(0, 3, 1, 2))
    assert float((y.double() - ref).norm() / ref.norm()) < 1e-5


def test_resnet101_infer_vs_torchvision():
    tv = pytest.importorskip("torchvision")
    P = si.make_params(om.resnet_spec(om.RESNET101_LAYERS))
    m = tv.models.resnet101().double().eval()
    _to_tv(P, m, _rn_rename)
    x = si.normal((1, 64, 64, 3), 4)
    y = om.resnet_infer(P, x, om.RESNET101_LAYERS)
    with torch.no_grad():
        ref = m(x.double().permute(0, 3, 1, 2))
    assert float((y.double() - ref).norm() / ref.norm()) < 1e-5
