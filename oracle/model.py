"""CPU ORACLE (test infrastructure only) — plain fp64 forward/backward of the workload models.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this module. It shares no code with the CUDA path (paper_conf_eurosys_stratimk24_b200/).

What it computes. Orion's numeric outputs have a plain definition independent of scheduling
(§5.1: Orion only decides *when* each client's kernels launch; stream order keeps each
client's data dependencies). So the oracle is each client's model written out with
PyTorch/TorchVision semantics, which is what the paper ran (TorchVision ResNet50 /
MobileNet-v2, full precision):
  * every op computes in float64 with plain torch CPU primitives (a conv, a matmul, a sum);
  * every op's output is rounded to the GPU's storage dtype (float32) before the next op uses it,
    exactly as the unfused GPU op stream materialises it (DESIGN.md §3 R22-R24);
  * backward passes are written out op by op (no autograd), in the reverse order of the forward.
Layouts follow the GPU's HBM layout so buffers can be compared element by element:
activations NHWC, conv weights OHWI ([Cout, kh, kw, Cin/groups]), linear weights [out, in].

Pins (tests/test_oracle_model.py): explicit-loop brute force of every forward op on tiny shapes,
central finite differences (fp64) of every backward op, closed forms (BN output moments, CE of
uniform logits = log C, MSE), and model-level gradients against fp64 autograd of the same forward.
"""
import math

import torch
import torch.nn.functional as F

F64 = torch.float64
F32 = torch.float32


def _r(t):
    """Round an fp64 result to the fp32 storage dtype (the unfused GPU op writes fp32)."""
    return t.to(F32)


def _d(t):
    return t.to(F64)


def _nchw(x):   # NHWC -> NCHW view for torch primitives
    return x.permute(0, 3, 1, 2)


def _nhwc(x):
    return x.permute(0, 2, 3, 1).contiguous()


def _w_oihw(w):  # OHWI -> OIHW
    return w.permute(0, 3, 1, 2)


# ----------------------------------------------------------------------------------- linear
def linear_fwd(x, w, b):
    """y = x W^T + b  (torch.nn.Linear). x [B, in], w [out, in], b [out]."""
    return _r(_d(x) @ _d(w).t() + (_d(b) if b is not None else 0.0))


def linear_bwd(x, w, dy):
    """dx = dy W, dW = dy^T x, db = sum_b dy."""
    dyd = _d(dy)
    return _r(dyd @ _d(w)), _r(dyd.t() @ _d(x)), _r(dyd.sum(0))


# ------------------------------------------------------------------------------------- conv
def conv2d_fwd(x, w, stride=1, pad=0, groups=1):
    """Conv2d, zero padding, no bias (TorchVision convs are bias-free). x NHWC, w OHWI."""
    y = F.conv2d(_nchw(_d(x)), _w_oihw(_d(w)), None, stride, pad, 1, groups)
    return _r(_nhwc(y))


def conv2d_bwd_data(dy, w, x_shape, stride=1, pad=0, groups=1):
    dx = torch.nn.grad.conv2d_input((x_shape[0], x_shape[3], x_shape[1], x_shape[2]), _w_oihw(_d(w)),
                                    _nchw(_d(dy)), stride, pad, 1, groups)
    return _r(_nhwc(dx))


def conv2d_bwd_weight(x, dy, w_shape, stride=1, pad=0, groups=1):
    o, kh, kw, ig = w_shape
    dw = torch.nn.grad.conv2d_weight(_nchw(_d(x)), (o, ig, kh, kw), _nchw(_d(dy)), stride, pad, 1, groups)
    return _r(dw.permute(0, 2, 3, 1).contiguous())


# --------------------------------------------------------------------------------------- BN
def bn_eval(x, gamma, beta, rmean, rvar, eps=1e-5):
    """BatchNorm2d eval: (x - rm) / sqrt(rv + eps) * gamma + beta, per channel (last dim)."""
    inv = 1.0 / torch.sqrt(_d(rvar) + eps)
    return _r((_d(x) - _d(rmean)) * inv * _d(gamma) + _d(beta))


def bn_train_fwd(x, gamma, beta, rmean, rvar, eps=1e-5, momentum=0.1):
    """BatchNorm2d train: normalise with the batch mean and biased variance; update running stats
    with momentum and the *unbiased* variance (torch semantics). Returns y, mean, invstd, rm', rv'."""
    xd = _d(x)
    c = x.shape[-1]
    flat = xd.reshape(-1, c)
    n = flat.shape[0]
    mean = flat.mean(0)
    var = ((flat - mean) ** 2).mean(0)
    invstd = 1.0 / torch.sqrt(var + eps)
    y = (xd - mean) * invstd * _d(gamma) + _d(beta)
    rm = (1 - momentum) * _d(rmean) + momentum * mean
    rv = (1 - momentum) * _d(rvar) + momentum * var * n / (n - 1)
    return _r(y), _r(mean), _r(invstd), _r(rm), _r(rv)


def bn_bwd_abs(x, dy, mean, invstd):
    """Absolute-term sums of bn_bwd's parameter gradients: sum |dy * xhat| and sum |dy| per
    channel. Not a result of the method: the scale of the rounding-error bound of each gradient
    element (|fl(sum t) - sum t| <= c u sum |t|), used by the parity tests' error model
    (DESIGN.md §8)."""
    c = x.shape[-1]
    xhat = (_d(x).reshape(-1, c) - _d(mean)) * _d(invstd)
    dyd = _d(dy).reshape(-1, c).abs()
    return (dyd * xhat.abs()).sum(0), dyd.sum(0)


def conv2d_bwd_weight_abs(x, dy, w_shape, stride=1, pad=0, groups=1):
    """sum |x| |dy| over the same (image, tap) pairs as conv2d_bwd_weight: its error-bound scale."""
    o, kh, kw, ig = w_shape
    dw = torch.nn.grad.conv2d_weight(_nchw(_d(x).abs()), (o, ig, kh, kw), _nchw(_d(dy).abs()), stride, pad, 1, groups)
    return dw.permute(0, 2, 3, 1).contiguous()


def bn_bwd(x, dy, gamma, mean, invstd):
    """Backward of training-mode BN given the saved (fp32) batch mean / invstd.
    xhat = (x-mean)*invstd; dbeta = sum dy; dgamma = sum dy*xhat;
    dx = gamma*invstd/N * (N dy - dbeta - xhat dgamma)."""
    c = x.shape[-1]
    xd = _d(x).reshape(-1, c)
    dyd = _d(dy).reshape(-1, c)
    n = xd.shape[0]
    xhat = (xd - _d(mean)) * _d(invstd)
    dbeta = dyd.sum(0)
    dgamma = (dyd * xhat).sum(0)
    dx = _d(gamma) * _d(invstd) / n * (n * dyd - dbeta - xhat * dgamma)
    return _r(dx.reshape(x.shape)), _r(dgamma), _r(dbeta)


# ------------------------------------------------------------------------------ elementwise
def relu(x):
    return _r(torch.clamp(_d(x), min=0.0))


def relu_bwd(x, dy):
    """Gradient passes where x > 0 (torch threshold_backward)."""
    return _r(torch.where(_d(x) > 0, _d(dy), torch.zeros((), dtype=F64)))


def relu6(x):
    return _r(torch.clamp(_d(x), 0.0, 6.0))


def relu6_bwd(x, dy):
    """hardtanh_backward(0, 6): gradient passes where 0 < x < 6."""
    xd = _d(x)
    return _r(torch.where((xd > 0) & (xd < 6), _d(dy), torch.zeros((), dtype=F64)))


def add(a, b):
    return _r(_d(a) + _d(b))


# ---------------------------------------------------------------------------------- pooling
def maxpool3x3s2(x):
    """MaxPool2d(3, stride 2, padding 1), -inf padding. NHWC."""
    y = F.max_pool2d(_nchw(_d(x)), 3, 2, 1)
    return _r(_nhwc(y))


def avgpool_fwd(x):
    """Global average pool (AdaptiveAvgPool2d(1) + flatten): [N,H,W,C] -> [N,C]."""
    return _r(_d(x).mean(dim=(1, 2)))


def avgpool_bwd(dy, x_shape):
    n, h, w, c = x_shape
    return _r((_d(dy) / (h * w)).reshape(n, 1, 1, c).expand(n, h, w, c).contiguous())


# ------------------------------------------------------------------------------------ losses
def ce_fwd_bwd(z, labels):
    """Cross entropy, mean over batch: L = mean_i(logsumexp(z_i) - z_i[y_i]);
    dz = (softmax(z) - onehot(y)) / B."""
    zd = _d(z)
    b = zd.shape[0]
    lse = torch.logsumexp(zd, dim=1)
    loss = (lse - zd[torch.arange(b), labels.long()]).mean()
    p = torch.exp(zd - lse[:, None])
    p[torch.arange(b), labels.long()] -= 1.0
    return _r(loss), _r(p / b)


def mse_fwd_bwd(y, t):
    """MSE, mean over all elements: L = mean((y-t)^2); dy = 2 (y-t) / numel."""
    diff = _d(y) - _d(t)
    return _r((diff ** 2).mean()), _r(2.0 * diff / diff.numel())


# ---------------------------------------------------------------------------------- optimizer
def sgd(p, g, v, lr, momentum, first):
    """torch.optim.SGD (dampening 0, no weight decay): v <- g (first step) else mu v + g;
    p <- p - lr v. With momentum == 0 the buffer is unused: p <- p - lr g."""
    if momentum == 0.0:
        return _r(_d(p) - lr * _d(g)), v
    vn = _d(g) if first else momentum * _d(v) + _d(g)
    return _r(_d(p) - lr * _r(vn).to(F64)), _r(vn)


# ================================================================================== models
# Parameter specs: ordered list of (name, shape, init). `init` names a distribution that the
# seeded generator (synth/inputs.py) draws from; the oracle never draws random numbers itself.

def mlp_spec(width=512, layers=3):
    spec = []
    for i in range(layers):
        spec.append((f"fc{i}.w", (width, width), ("uniform_fan_in", width)))
        spec.append((f"fc{i}.b", (width,), ("uniform_fan_in", width)))
    return spec


def mlp_fwd(P, x, layers=3, keep=False):
    """Toy MLP (BASELINE config 1): Linear-ReLU-Linear-ReLU-Linear."""
    acts = [x]
    h = x
    for i in range(layers):
        h = linear_fwd(h, P[f"fc{i}.w"], P[f"fc{i}.b"])
        acts.append(h)
        if i < layers - 1:
            h = relu(h)
            acts.append(h)
    return (h, acts) if keep else h


def mlp_train_step(P, x, t, lr=0.01, layers=3):
    """One SGD(momentum 0) step with MSE loss. Returns (loss, new params)."""
    y, acts = mlp_fwd(P, x, layers, keep=True)
    loss, dy = mse_fwd_bwd(y, t)
    grads = {}
    # acts: [x, z0, h0, z1, h1, z2]
    for i in reversed(range(layers)):
        inp = acts[2 * i]
        dx, dw, db = linear_bwd(inp, P[f"fc{i}.w"], dy)
        grads[f"fc{i}.w"], grads[f"fc{i}.b"] = dw, db
        if i > 0:
            dy = relu_bwd(acts[2 * i - 1], dx)
    newP = {k: sgd(P[k], grads[k], None, lr, 0.0, True)[0] for k in P}
    return loss, newP, grads


# ------------------------------------------------------------------------------ ResNet-50
RESNET50_LAYERS = [(64, 3, 1), (128, 4, 2), (256, 6, 2), (512, 3, 2)]   # (width, blocks, stride)
RESNET101_LAYERS = [(64, 3, 1), (128, 4, 2), (256, 23, 2), (512, 3, 2)]


def _bn_spec(name, c, eval_stats):
    s = [(f"{name}.gamma", (c,), ("const", 1.0)), (f"{name}.beta", (c,), ("const", 0.0))]
    if eval_stats:
        s += [(f"{name}.rmean", (c,), ("normal", 0.1)), (f"{name}.rvar", (c,), ("uniform", 0.5, 1.5))]
    else:
        s += [(f"{name}.rmean", (c,), ("const", 0.0)), (f"{name}.rvar", (c,), ("const", 1.0))]
    return s


def _conv_spec(name, cout, k, cin_g):
    # kaiming_normal_(mode='fan_out', relu): std = sqrt(2 / (cout * k * k))
    return [(f"{name}.w", (cout, k, k, cin_g), ("kaiming_fan_out", cout * k * k))]


def resnet_spec(layers=RESNET50_LAYERS, num_classes=1000, eval_stats=True):
    s = _conv_spec("conv1", 64, 7, 3) + _bn_spec("bn1", 64, eval_stats)
    cin = 64
    for li, (w, nb, stride) in enumerate(layers):
        for bi in range(nb):
            p = f"layer{li + 1}.{bi}"
            s += _conv_spec(f"{p}.conv1", w, 1, cin) + _bn_spec(f"{p}.bn1", w, eval_stats)
            s += _conv_spec(f"{p}.conv2", w, 3, w) + _bn_spec(f"{p}.bn2", w, eval_stats)
            s += _conv_spec(f"{p}.conv3", 4 * w, 1, w) + _bn_spec(f"{p}.bn3", 4 * w, eval_stats)
            if bi == 0:
                s += _conv_spec(f"{p}.down", 4 * w, 1, cin) + _bn_spec(f"{p}.downbn", 4 * w, eval_stats)
            cin = 4 * w
    s += [("fc.w", (num_classes, cin), ("uniform_fan_in", cin)), ("fc.b", (num_classes,), ("uniform_fan_in", cin))]
    return s


def resnet_infer(P, x, layers=RESNET50_LAYERS):
    """TorchVision ResNet v1.5 (stride on the 3x3), eval-mode BN. x NHWC [N,H,W,3] -> logits [N,1000]."""
    def cbr(h, name, bn, stride, pad, act=True):
        h = conv2d_fwd(h, P[f"{name}.w"], stride, pad)
        h = bn_eval(h, P[f"{bn}.gamma"], P[f"{bn}.beta"], P[f"{bn}.rmean"], P[f"{bn}.rvar"])
        return relu(h) if act else h
    h = cbr(x, "conv1", "bn1", 2, 3)
    h = maxpool3x3s2(h)
    for li, (w, nb, stride) in enumerate(layers):
        for bi in range(nb):
            p = f"layer{li + 1}.{bi}"
            s = stride if bi == 0 else 1
            o = cbr(h, f"{p}.conv1", f"{p}.bn1", 1, 0)
            o = cbr(o, f"{p}.conv2", f"{p}.bn2", s, 1)
            o = cbr(o, f"{p}.conv3", f"{p}.bn3", 1, 0, act=False)
            idn = cbr(h, f"{p}.down", f"{p}.downbn", s, 0, act=False) if bi == 0 else h
            h = relu(add(o, idn))
    h = avgpool_fwd(h)
    return linear_fwd(h, P["fc.w"], P["fc.b"])


# ---------------------------------------------------------------------------- MobileNetV2
MNV2_SETTINGS = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2), (6, 96, 3, 1),
                 (6, 160, 3, 2), (6, 320, 1, 1)]   # torchvision (t, c, n, s)


def mnv2_blocks(width_mult=1.0):
    """Block list: (name, cin, hidden, cout, stride, expand, residual)."""
    blocks = []
    cin = 32
    i = 1
    for t, c, n, s in MNV2_SETTINGS:
        for j in range(n):
            stride = s if j == 0 else 1
            hidden = cin * t
            blocks.append((f"features.{i}", cin, hidden, c, stride, t != 1, stride == 1 and cin == c))
            cin = c
            i += 1
    return blocks


def mnv2_spec(num_classes=1000, eval_stats=False):
    """eval_stats: seeded running statistics (the inference clients, reading R22) instead of torch's
    training start (0, 1)."""
    e = eval_stats
    s = _conv_spec("features.0", 32, 3, 3) + _bn_spec("features.0.bn", 32, e)
    for name, cin, hid, cout, stride, expand, res in mnv2_blocks():
        if expand:
            s += _conv_spec(f"{name}.expand", hid, 1, cin) + _bn_spec(f"{name}.expand_bn", hid, e)
        s += _conv_spec(f"{name}.dw", hid, 3, 1) + _bn_spec(f"{name}.dw_bn", hid, e)
        s += _conv_spec(f"{name}.project", cout, 1, hid) + _bn_spec(f"{name}.project_bn", cout, e)
    s += _conv_spec("features.18", 1280, 1, 320) + _bn_spec("features.18.bn", 1280, e)
    # torchvision MobileNetV2 classifier init: normal(0, 0.01), bias zeros
    s += [("classifier.w", (num_classes, 1280), ("normal", 0.01)), ("classifier.b", (num_classes,), ("const", 0.0))]
    return s


def mnv2_infer(P, x):
    """TorchVision MobileNetV2 inference (eval-mode BN, ReLU6, dropout inactive): x NHWC [N,H,W,3] ->
    logits. A best-effort inference client of the inf-inf configuration (Table 1 b4)."""
    def cb(h, cname, bname, k, stride, groups, act):
        h = conv2d_fwd(h, P[f"{cname}.w"], stride, k // 2, groups)
        h = bn_eval(h, P[f"{bname}.gamma"], P[f"{bname}.beta"], P[f"{bname}.rmean"], P[f"{bname}.rvar"])
        return relu6(h) if act else h
    h = cb(x, "features.0", "features.0.bn", 3, 2, 1, True)
    for name, cin, hid, cout, stride, expand, res in mnv2_blocks():
        inp = h
        if expand:
            h = cb(h, f"{name}.expand", f"{name}.expand_bn", 1, 1, 1, True)
        h = cb(h, f"{name}.dw", f"{name}.dw_bn", 3, stride, hid, True)
        h = cb(h, f"{name}.project", f"{name}.project_bn", 1, 1, 1, False)
        if res:
            h = add(h, inp)
    h = cb(h, "features.18", "features.18.bn", 1, 1, 1, True)
    return linear_fwd(avgpool_fwd(h), P["classifier.w"], P["classifier.b"])


def mnv2_trainable(spec):
    """Names of the parameters SGD updates (BN running stats are buffers, not parameters)."""
    return [n for n, _, _ in spec if not (n.endswith(".rmean") or n.endswith(".rvar"))]


def mnv2_train_step(P, V, x, labels, first, lr=0.01, momentum=0.9, eps=1e-5, bn_momentum=0.1, masks=None, trace=None):
    """One training iteration of torchvision MobileNetV2 (dropout p=0, reading R22) with
    CE loss and SGD(momentum). P: params + BN running stats (dict of fp32 tensors);
    V: momentum buffers (dict). Returns (loss, newP, newV, grads).

    masks (optional): {bn name: fp32 tensor} — the values on which the ReLU6 backward takes its
    pass/stop decision (0 < y < 6). A decision is an integer decided by floating point; to compare
    a fp32 GPU backward with this fp64 oracle both must decide on the same value, so
    parity tests pass the GPU's own BN outputs here, after auditing them against the oracle's own
    (trace["bn_out"]). All arithmetic stays the oracle's.

    trace (optional dict, test instrumentation): filled with "bn_out" {bn name: the oracle's own BN
    output, on which its free-running ReLU6 decides} and "abs" {gradient name: the absolute-term sum
    of every gradient element, the scale of its rounding-error bound}."""
    newP = dict(P)
    if trace is not None:
        trace.setdefault("bn_out", {})
        trace.setdefault("abs", {})

    def conv_bn(h, cname, bname, k, stride, groups, act):
        z = conv2d_fwd(h, P[f"{cname}.w"], stride, k // 2, groups)
        y, mean, invstd, rm, rv = bn_train_fwd(z, P[f"{bname}.gamma"], P[f"{bname}.beta"],
                                               P[f"{bname}.rmean"], P[f"{bname}.rvar"], eps, bn_momentum)
        newP[f"{bname}.rmean"], newP[f"{bname}.rvar"] = rm, rv
        if trace is not None:
            trace["bn_out"][bname] = y
        rec = (cname, bname, k, stride, groups, act, h, z, y, mean, invstd)
        return (relu6(y) if act else y), rec

    g = {}

    def conv_bn_bwd(rec, dout, need_dx=True):
        cname, bname, k, stride, groups, act, hin, z, y, mean, invstd = rec
        dy = relu6_bwd(masks[bname] if masks is not None else y, dout) if act else dout
        dz, g[f"{bname}.gamma"], g[f"{bname}.beta"] = bn_bwd(z, dy, P[f"{bname}.gamma"], mean, invstd)
        w = P[f"{cname}.w"]
        g[f"{cname}.w"] = conv2d_bwd_weight(hin, dz, tuple(w.shape), stride, k // 2, groups)
        if trace is not None:
            trace["abs"][f"{bname}.gamma"], trace["abs"][f"{bname}.beta"] = bn_bwd_abs(z, dy, mean, invstd)
            trace["abs"][f"{cname}.w"] = conv2d_bwd_weight_abs(hin, dz, tuple(w.shape), stride, k // 2, groups)
        return conv2d_bwd_data(dz, w, tuple(hin.shape), stride, k // 2, groups) if need_dx else None

    # ---- forward
    h, stem = conv_bn(x, "features.0", "features.0.bn", 3, 2, 1, True)
    recs = []
    for name, cin, hid, cout, stride, expand, res in mnv2_blocks():
        inp = h
        r = {}
        if expand:
            h, r["expand"] = conv_bn(h, f"{name}.expand", f"{name}.expand_bn", 1, 1, 1, True)
        h, r["dw"] = conv_bn(h, f"{name}.dw", f"{name}.dw_bn", 3, stride, hid, True)
        h, r["project"] = conv_bn(h, f"{name}.project", f"{name}.project_bn", 1, 1, 1, False)
        if res:
            h = add(h, inp)
        recs.append((res, r))
    h, last = conv_bn(h, "features.18", "features.18.bn", 1, 1, 1, True)
    feat_shape = tuple(h.shape)
    pooled = avgpool_fwd(h)
    logits = linear_fwd(pooled, P["classifier.w"], P["classifier.b"])
    loss, dlogits = ce_fwd_bwd(logits, labels)

    # ---- backward (reverse op order)
    dpooled, g["classifier.w"], g["classifier.b"] = linear_bwd(pooled, P["classifier.w"], dlogits)
    if trace is not None:
        trace["abs"]["classifier.w"] = _d(dlogits).abs().t() @ _d(pooled).abs()
        trace["abs"]["classifier.b"] = _d(dlogits).abs().sum(0)
    dh = avgpool_bwd(dpooled, feat_shape)
    dh = conv_bn_bwd(last, dh)
    for res, r in reversed(recs):
        d = conv_bn_bwd(r["project"], dh)
        d = conv_bn_bwd(r["dw"], d)
        if "expand" in r:
            d = conv_bn_bwd(r["expand"], d)
        dh = add(d, dh) if res else d
    conv_bn_bwd(stem, dh, need_dx=False)

    # ---- optimizer
    newV = {}
    for n in sorted(g):
        newP[n], newV[n] = sgd(P[n], g[n], V.get(n), lr, momentum, first)
    return loss, newP, newV, g


# ------------------------------------------------------------------- max-pool backward
def maxpool3x3s2_bwd(x, dy):
    """Backward of MaxPool2d(3, 2, 1): each output's gradient goes to the first maximum of its
    window in row-major (u, v) order; contributions to one input add up. NHWC."""
    xd, dyd = _d(x), _d(dy)
    n, h, w, c = x.shape
    p, q = dy.shape[1], dy.shape[2]
    xp = torch.full((n, h + 2, w + 2, c), -math.inf, dtype=F64)
    xp[:, 1:h + 1, 1:w + 1, :] = xd
    best = torch.full((n, p, q, c), -math.inf, dtype=F64)
    arg = torch.zeros((n, p, q, c), dtype=torch.long)
    for u in range(3):
        for v in range(3):
            win = xp[:, u:u + 2 * p:2, v:v + 2 * q:2, :][:, :p, :q, :]
            take = win > best                       # strict: the first maximum wins ties
            best = torch.where(take, win, best)
            arg = torch.where(take, torch.full_like(arg, u * 3 + v), arg)
    dxp = torch.zeros((n, h + 2, w + 2, c), dtype=F64)
    for u in range(3):
        for v in range(3):
            sel = torch.where(arg == u * 3 + v, dyd, torch.zeros((), dtype=F64))
            dxp[:, u:u + 2 * p:2, v:v + 2 * q:2, :][:, :p, :q, :] += sel
    return _r(dxp[:, 1:h + 1, 1:w + 1, :])


# -------------------------------------------------------------------- ResNet training
def resnet_train_step(P, V, x, labels, first, layers=RESNET50_LAYERS, lr=0.01, momentum=0.9, eps=1e-5,
                      bn_momentum=0.1, masks=None, trace=None):
    """One training iteration of TorchVision ResNet v1.5 (train-mode BN, CE, SGD momentum), the
    BE client of BASELINE config 3 (ResNet-50, batch 64) and HP of config 4 (ResNet-101).
    Ops in PyTorch eager order, each rounded to fp32 (R22-R24). masks (optional): {name: fp32
    tensor} of the values the GPU's ReLU backward decides on (its BN / residual-sum outputs), as in
    mnv2_train_step; the max-pool backward then also picks its first maxima on
    relu(masks["bn1"]), the GPU's own max-pool input. trace (optional dict): filled with "relu_in"
    {name: the oracle's own ReLU input} and "abs" {gradient: absolute-term sums}, as in
    mnv2_train_step. Returns (loss, newP, newV, grads)."""
    newP = dict(P)
    g = {}
    if trace is not None:
        trace.setdefault("relu_in", {})
        trace.setdefault("abs", {})

    def cb(h, cname, bname, stride, pad):
        z = conv2d_fwd(h, P[f"{cname}.w"], stride, pad)
        y, mean, invstd, rm, rv = bn_train_fwd(z, P[f"{bname}.gamma"], P[f"{bname}.beta"],
                                               P[f"{bname}.rmean"], P[f"{bname}.rvar"], eps, bn_momentum)
        newP[f"{bname}.rmean"], newP[f"{bname}.rvar"] = rm, rv
        return y, (cname, bname, stride, pad, h, z, mean, invstd)

    def cb_bwd(rec, dy, need_dx=True):
        cname, bname, stride, pad, hin, z, mean, invstd = rec
        dz, g[f"{bname}.gamma"], g[f"{bname}.beta"] = bn_bwd(z, dy, P[f"{bname}.gamma"], mean, invstd)
        w = P[f"{cname}.w"]
        g[f"{cname}.w"] = conv2d_bwd_weight(hin, dz, tuple(w.shape), stride, pad)
        if trace is not None:
            trace["abs"][f"{bname}.gamma"], trace["abs"][f"{bname}.beta"] = bn_bwd_abs(z, dy, mean, invstd)
            trace["abs"][f"{cname}.w"] = conv2d_bwd_weight_abs(hin, dz, tuple(w.shape), stride, pad)
        return conv2d_bwd_data(dz, w, tuple(hin.shape), stride, pad) if need_dx else None

    def m(name, val):
        if trace is not None:
            trace["relu_in"][name] = val
        return masks[name] if masks is not None else val

    # ---- forward
    y, stem = cb(x, "conv1", "bn1", 2, 3)
    a = relu(y)
    mp = maxpool3x3s2(a)
    h = mp
    blocks = []
    for li, (w, nb, stride) in enumerate(layers):
        for bi in range(nb):
            p = f"layer{li + 1}.{bi}"
            s = stride if bi == 0 else 1
            y1, r1 = cb(h, f"{p}.conv1", f"{p}.bn1", 1, 0)
            a1 = relu(y1)
            y2, r2 = cb(a1, f"{p}.conv2", f"{p}.bn2", s, 1)
            a2 = relu(y2)
            y3, r3 = cb(a2, f"{p}.conv3", f"{p}.bn3", 1, 0)
            if bi == 0:
                idn, rd = cb(h, f"{p}.down", f"{p}.downbn", s, 0)
            else:
                idn, rd = h, None
            sm = add(y3, idn)
            out = relu(sm)
            blocks.append((p, r1, y1, r2, y2, r3, rd, sm))
            h = out
    feat_shape = tuple(h.shape)
    pooled = avgpool_fwd(h)
    logits = linear_fwd(pooled, P["fc.w"], P["fc.b"])
    loss, dlogits = ce_fwd_bwd(logits, labels)

    # ---- backward (reverse op order)
    dpooled, g["fc.w"], g["fc.b"] = linear_bwd(pooled, P["fc.w"], dlogits)
    if trace is not None:
        trace["abs"]["fc.w"] = _d(dlogits).abs().t() @ _d(pooled).abs()
        trace["abs"]["fc.b"] = _d(dlogits).abs().sum(0)
    dh = avgpool_bwd(dpooled, feat_shape)
    for p, r1, y1, r2, y2, r3, rd, sm in reversed(blocks):
        dsm = relu_bwd(m(f"{p}.sum", sm), dh)
        d = cb_bwd(r3, dsm)
        d = relu_bwd(m(f"{p}.bn2", y2), d)
        d = cb_bwd(r2, d)
        d = relu_bwd(m(f"{p}.bn1", y1), d)
        d = cb_bwd(r1, d)
        didn = cb_bwd(rd, dsm) if rd is not None else dsm
        dh = add(d, didn)
    da = maxpool3x3s2_bwd(relu(masks["bn1"]) if masks is not None else a, dh)
    dy = relu_bwd(m("bn1", y), da)
    cb_bwd(stem, dy, need_dx=False)

    newV = {}
    for n in sorted(g):
        newP[n], newV[n] = sgd(P[n], g[n], V.get(n), lr, momentum, first)
    return loss, newP, newV, g


def resnet_train_spec(layers=RESNET50_LAYERS, num_classes=1000):
    """Training ResNet: BN running stats start at torch's defaults (mean 0, var 1)."""
    return resnet_spec(layers, num_classes, eval_stats=False)


# ============================================================================ BERT (bf16)
# HP of BASELINE config 3: BERT-base inference, batch 8, sequence 128, bf16 (HuggingFace
# BertModel as PyTorch eager runs it with the model cast to bfloat16; readings R22, R29-R31 in
# DESIGN.md §3). Every op computes in float64 from its bf16 inputs and rounds its output once to
# bf16 (round-to-nearest-even), as the unfused GPU op stream materialises it. `store` selects the
# storage dtype so the pins can run the same code unrounded (float64) against HF's fp64 model.
BF16 = torch.bfloat16


def _s(t, store):
    return t.to(store)


def bert_spec(layers=12, hidden=768, heads=12, ffn=3072, vocab=30522, max_pos=512, types=2):
    """Parameter spec (names, shapes, init). Linear weights [out, in]. Init (reading R22): every
    weight, embedding and bias N(0, 0.02); LayerNorm gamma U[0.9, 1.1], beta N(0, 0.02) (non-zero
    biases / non-unit gammas so that every term of every op is exercised)."""
    n = ("normal", 0.02)
    s = [("emb.word", (vocab, hidden), n), ("emb.pos", (max_pos, hidden), n), ("emb.type", (types, hidden), n),
         ("emb.ln.gamma", (hidden,), ("uniform", 0.9, 1.1)), ("emb.ln.beta", (hidden,), n)]
    for i in range(layers):
        p = f"layer{i}"
        for nm, o, k in (("q", hidden, hidden), ("k", hidden, hidden), ("v", hidden, hidden), ("o", hidden, hidden),
                         ("ffn1", ffn, hidden), ("ffn2", hidden, ffn)):
            s += [(f"{p}.{nm}.w", (o, k), n), (f"{p}.{nm}.b", (o,), n)]
        for ln in ("ln1", "ln2"):
            s += [(f"{p}.{ln}.gamma", (hidden,), ("uniform", 0.9, 1.1)), (f"{p}.{ln}.beta", (hidden,), n)]
    return s


def bert_embed(ids, word, pos, typ, store=BF16):
    """embeddings = word[ids] + type[0] + pos[s] (token type 0 everywhere, no padding: R22),
    summed in fp64 and rounded once. ids [B, S] -> [B, S, H]."""
    b, sq = ids.shape
    e = _d(word)[ids.long()] + _d(typ)[0] + _d(pos)[:sq][None, :, :]
    return _s(e, store)


def layernorm(x, gamma, beta, eps=1e-12, store=BF16):
    """LayerNorm over the last dim: (x - mean) / sqrt(var + eps) * gamma + beta, biased var."""
    xd = _d(x)
    mean = xd.mean(-1, keepdim=True)
    var = ((xd - mean) ** 2).mean(-1, keepdim=True)
    return _s((xd - mean) / torch.sqrt(var + eps) * _d(gamma) + _d(beta), store)


def linear_any(x, w, b, store=BF16):
    """y = x W^T + b over the last dim, fp64 accumulation, one rounding."""
    return _s(_d(x) @ _d(w).t() + _d(b), store)


def gelu(x, store=BF16):
    """GELU, exact erf form: 0.5 x (1 + erf(x / sqrt 2)) (HF "gelu")."""
    xd = _d(x)
    return _s(0.5 * xd * (1.0 + torch.erf(xd / math.sqrt(2.0))), store)


def add_any(a, b, store=BF16):
    return _s(_d(a) + _d(b), store)


def attention(q, k, v, heads, store=BF16):
    """Multi-head scaled dot-product attention without mask (R22): per batch b and head h,
    O = softmax(Q K^T / sqrt(d)) V with Q, K, V the head's d = H/heads columns of [B, S, H].
    One op (the fused SDPA kernel PyTorch dispatches), fp64 inside, one rounding of O."""
    b, sq, hd = q.shape
    d = hd // heads
    Q = _d(q).view(b, sq, heads, d).permute(0, 2, 1, 3)
    K = _d(k).view(b, sq, heads, d).permute(0, 2, 1, 3)
    Vv = _d(v).view(b, sq, heads, d).permute(0, 2, 1, 3)
    sc = Q @ K.transpose(-1, -2) / math.sqrt(d)
    pr = torch.softmax(sc, dim=-1)
    o = (pr @ Vv).permute(0, 2, 1, 3).reshape(b, sq, hd)
    return _s(o, store)


def bert_infer(P, ids, layers=12, heads=12, store=BF16):
    """BertModel forward (no pooler): last hidden state [B, S, H] in `store`. P holds the
    parameters already in the model dtype (bf16, or fp64 for the pins)."""
    h = bert_embed(ids, P["emb.word"], P["emb.pos"], P["emb.type"], store)
    h = layernorm(h, P["emb.ln.gamma"], P["emb.ln.beta"], store=store)
    for i in range(layers):
        p = f"layer{i}"
        q = linear_any(h, P[f"{p}.q.w"], P[f"{p}.q.b"], store)
        k = linear_any(h, P[f"{p}.k.w"], P[f"{p}.k.b"], store)
        v = linear_any(h, P[f"{p}.v.w"], P[f"{p}.v.b"], store)
        a = attention(q, k, v, heads, store)
        o = linear_any(a, P[f"{p}.o.w"], P[f"{p}.o.b"], store)
        h1 = layernorm(add_any(o, h, store), P[f"{p}.ln1.gamma"], P[f"{p}.ln1.beta"], store=store)
        f = gelu(linear_any(h1, P[f"{p}.ffn1.w"], P[f"{p}.ffn1.b"], store), store)
        f2 = linear_any(f, P[f"{p}.ffn2.w"], P[f"{p}.ffn2.b"], store)
        h = layernorm(add_any(f2, h1, store), P[f"{p}.ln2.gamma"], P[f"{p}.ln2.beta"], store=store)
    return h


def to_model_dtype(P, dtype=BF16):
    """Cast drawn parameters to the model dtype (model.to(torch.bfloat16))."""
    return {k: v.to(dtype) for k, v in P.items()}


# ------------------------------------------------------------------------- small helpers
def count_flops_conv(n, ho, wo, cout, k, cin_g):
    return 2 * n * ho * wo * cout * k * k * cin_g


def out_hw(h, k, s, p):
    return (h + 2 * p - k) // s + 1


def logsumexp_uniform(c):
    return math.log(c)


# ------------------------------------------------------------------------------- col2im
def col2im(col, x_shape, R, S, stride, pad):
    """col2im (the adjoint of im2col): dx[n,h,w,c] = sum over (p,q,r,s) with h = p*stride - pad + r,
    w = q*stride - pad + s of col[n,p,q,r,s,c]. col [N*P*Q, R*S*C] (rows (n,p,q), columns (r,s,c)
    with c fastest), dx NHWC. With col = dy W (W as [K, R*S*C]) this is the data gradient of a
    convolution, the form liborion uses for strided convs. torch's fold = col2im."""
    n, h, w, c = x_shape
    p, q = (h + 2 * pad - R) // stride + 1, (w + 2 * pad - S) // stride + 1
    cd = _d(col).view(n, p * q, R, S, c).permute(0, 4, 2, 3, 1).reshape(n, c * R * S, p * q)
    dx = F.fold(cd, (h, w), (R, S), padding=pad, stride=stride)
    return _r(_nhwc(dx))


# ============================================================ Transformer encoder training (fp32)
# BE of BASELINE config 4 (reading R32): torch.nn.TransformerEncoderLayer stack,
# post-LN (norm_first=False), ReLU FFN, dropout 0, batch_first; packed in-projection
# (in_proj_weight [3d, d], as nn.MultiheadAttention); MSE loss to a target; SGD(momentum).
# Every op computes in fp64 and rounds its output to fp32 (the unfused GPU op stream).

def encoder_spec(layers=6, d=512, ffn=2048):
    s = []
    for i in range(layers):
        p = f"enc{i}"
        s += [(f"{p}.in.w", (3 * d, d), ("uniform_fan_in", d)), (f"{p}.in.b", (3 * d,), ("const", 0.0)),
              (f"{p}.out.w", (d, d), ("uniform_fan_in", d)), (f"{p}.out.b", (d,), ("const", 0.0)),
              (f"{p}.ln1.gamma", (d,), ("const", 1.0)), (f"{p}.ln1.beta", (d,), ("const", 0.0)),
              (f"{p}.ff1.w", (ffn, d), ("uniform_fan_in", d)), (f"{p}.ff1.b", (ffn,), ("uniform_fan_in", d)),
              (f"{p}.ff2.w", (d, ffn), ("uniform_fan_in", ffn)), (f"{p}.ff2.b", (d,), ("uniform_fan_in", ffn)),
              (f"{p}.ln2.gamma", (d,), ("const", 1.0)), (f"{p}.ln2.beta", (d,), ("const", 0.0))]
    return s


def layernorm_fwd(x, gamma, beta, eps=1e-5):
    """LayerNorm over the last dim (biased variance). Returns y, mean, rstd (the saved statistics
    of the fused PyTorch kernel), each rounded to fp32."""
    xd = _d(x)
    mean = xd.mean(-1)
    var = ((xd - mean[..., None]) ** 2).mean(-1)
    rstd = 1.0 / torch.sqrt(var + eps)
    y = (xd - mean[..., None]) * rstd[..., None] * _d(gamma) + _d(beta)
    return _r(y), _r(mean), _r(rstd)


def layernorm_bwd(x, dy, gamma, mean, rstd):
    """Backward of LayerNorm from the saved fp32 mean / rstd: xhat = (x - mean) rstd;
    dgamma = sum_rows dy xhat; dbeta = sum_rows dy; dx = rstd (g - mean(g) - xhat mean(g xhat))
    with g = dy gamma."""
    xd, dyd = _d(x), _d(dy)
    xh = (xd - _d(mean)[..., None]) * _d(rstd)[..., None]
    g = dyd * _d(gamma)
    dx = _d(rstd)[..., None] * (g - g.mean(-1, keepdim=True) - xh * (g * xh).mean(-1, keepdim=True))
    red = tuple(range(x.dim() - 1))
    return _r(dx), _r((dyd * xh).sum(red)), _r(dyd.sum(red))


def mha_fwd(q, k, v, heads):
    """Scaled dot-product attention (no mask) per head on [B, S, H] views; fp32 output."""
    return attention(q, k, v, heads, store=F32)


def mha_bwd(q, k, v, do, heads):
    """Backward of softmax(Q K^T / sqrt d) V per head: P recomputed in fp64;
    dV = P^T dO, dP = dO V^T, dS = P (dP - rowsum(P dP)), dQ = dS K / sqrt d, dK = dS^T Q / sqrt d."""
    b, sq, hd = q.shape
    d = hd // heads

    def split(t):
        return _d(t).view(b, sq, heads, d).permute(0, 2, 1, 3)
    Q, K, V, dO = split(q), split(k), split(v), split(do)
    sc = Q @ K.transpose(-1, -2) / math.sqrt(d)
    P = torch.softmax(sc, dim=-1)
    dV = P.transpose(-1, -2) @ dO
    dP = dO @ V.transpose(-1, -2)
    dS = P * (dP - (P * dP).sum(-1, keepdim=True))
    dQ = dS @ K / math.sqrt(d)
    dK = dS.transpose(-1, -2) @ Q / math.sqrt(d)

    def merge(t):
        return _r(t.permute(0, 2, 1, 3).reshape(b, sq, hd))
    return merge(dQ), merge(dK), merge(dV)


def encoder_infer(P, x, layers=6, heads=8, eps=1e-5):
    """Forward of the post-LN encoder stack (reading R32) in fp32 storage: x [B, S, d] -> the last
    layer's output [B*S, d]. The "Transformer" inference client of the inf-inf configuration."""
    b, sq, dm = x.shape
    rows = b * sq
    h = x.reshape(rows, dm)
    for i in range(layers):
        p = f"enc{i}"
        qkv = linear_fwd(h, P[f"{p}.in.w"], P[f"{p}.in.b"])
        q, k, v = (qkv[:, j * dm:(j + 1) * dm].reshape(b, sq, dm) for j in range(3))
        a = mha_fwd(q, k, v, heads).reshape(rows, dm)
        s1 = add(h, linear_fwd(a, P[f"{p}.out.w"], P[f"{p}.out.b"]))
        h1, _, _ = layernorm_fwd(s1, P[f"{p}.ln1.gamma"], P[f"{p}.ln1.beta"], eps)
        f2 = linear_fwd(relu(linear_fwd(h1, P[f"{p}.ff1.w"], P[f"{p}.ff1.b"])), P[f"{p}.ff2.w"], P[f"{p}.ff2.b"])
        h, _, _ = layernorm_fwd(add(h1, f2), P[f"{p}.ln2.gamma"], P[f"{p}.ln2.beta"], eps)
    return h


def encoder_train_step(P, V, x, t, first, layers=6, heads=8, lr=0.01, momentum=0.9, eps=1e-5, masks=None, trace=None):
    """One training iteration of the post-LN encoder stack on x [B, S, d] with MSE to t.
    masks (optional): {name: fp32 tensor} — the values the GPU's ReLU backward decided on (its FFN
    pre-activations), as in the other training oracles. trace (optional dict):
    "relu_in" {name: the oracle's own FFN pre-activation} and "abs" {gradient: absolute-term sums}.
    Returns (loss, newP, newV, grads)."""
    b, sq, dm = x.shape
    rows = b * sq
    g = {}
    if trace is not None:
        trace.setdefault("relu_in", {})
        trace.setdefault("abs", {})

    def lin_abs(name, xin, dy):
        if trace is not None:
            trace["abs"][f"{name}.w"] = _d(dy).abs().t() @ _d(xin).abs()
            trace["abs"][f"{name}.b"] = _d(dy).abs().sum(0)

    def ln_abs(name, xin, dy, mean, rstd):
        if trace is not None:
            xh = ((_d(xin) - _d(mean)[..., None]) * _d(rstd)[..., None]).abs()
            red = tuple(range(xin.dim() - 1))
            trace["abs"][f"{name}.gamma"] = (_d(dy).abs() * xh).sum(red)
            trace["abs"][f"{name}.beta"] = _d(dy).abs().sum(red)
    recs = []
    h = x.reshape(rows, dm)
    for i in range(layers):
        p = f"enc{i}"
        qkv = linear_fwd(h, P[f"{p}.in.w"], P[f"{p}.in.b"])                 # [rows, 3d]
        q, k, v = (qkv[:, j * dm:(j + 1) * dm].reshape(b, sq, dm) for j in range(3))
        a = mha_fwd(q, k, v, heads).reshape(rows, dm)
        o = linear_fwd(a, P[f"{p}.out.w"], P[f"{p}.out.b"])
        s1 = add(h, o)
        h1, m1, r1 = layernorm_fwd(s1, P[f"{p}.ln1.gamma"], P[f"{p}.ln1.beta"], eps)
        f = linear_fwd(h1, P[f"{p}.ff1.w"], P[f"{p}.ff1.b"])
        fa = relu(f)
        f2 = linear_fwd(fa, P[f"{p}.ff2.w"], P[f"{p}.ff2.b"])
        s2 = add(h1, f2)
        h2, m2, r2 = layernorm_fwd(s2, P[f"{p}.ln2.gamma"], P[f"{p}.ln2.beta"], eps)
        recs.append((h, q, k, v, a, s1, h1, m1, r1, f, fa, s2, m2, r2))
        h = h2
    loss, dh = mse_fwd_bwd(h, t.reshape(rows, dm))
    for i in reversed(range(layers)):
        p = f"enc{i}"
        hin, q, k, v, a, s1, h1, m1, r1, f, fa, s2, m2, r2 = recs[i]
        ds2, g[f"{p}.ln2.gamma"], g[f"{p}.ln2.beta"] = layernorm_bwd(s2, dh, P[f"{p}.ln2.gamma"], m2, r2)
        ln_abs(f"{p}.ln2", s2, dh, m2, r2)
        dfa, g[f"{p}.ff2.w"], g[f"{p}.ff2.b"] = linear_bwd(fa, P[f"{p}.ff2.w"], ds2)
        lin_abs(f"{p}.ff2", fa, ds2)
        if trace is not None:
            trace["relu_in"][f"{p}.ff1"] = f
        df = relu_bwd(masks[f"{p}.ff1"] if masks is not None else f, dfa)
        dh1_ff, g[f"{p}.ff1.w"], g[f"{p}.ff1.b"] = linear_bwd(h1, P[f"{p}.ff1.w"], df)
        lin_abs(f"{p}.ff1", h1, df)
        dh1 = add(ds2, dh1_ff)
        ds1, g[f"{p}.ln1.gamma"], g[f"{p}.ln1.beta"] = layernorm_bwd(s1, dh1, P[f"{p}.ln1.gamma"], m1, r1)
        ln_abs(f"{p}.ln1", s1, dh1, m1, r1)
        da, g[f"{p}.out.w"], g[f"{p}.out.b"] = linear_bwd(a, P[f"{p}.out.w"], ds1)
        lin_abs(f"{p}.out", a, ds1)
        dq, dk, dv = mha_bwd(q, k, v, da.reshape(b, sq, dm), heads)
        dqkv = torch.cat([dq.reshape(rows, dm), dk.reshape(rows, dm), dv.reshape(rows, dm)], dim=1)
        dhin_attn, g[f"{p}.in.w"], g[f"{p}.in.b"] = linear_bwd(hin, P[f"{p}.in.w"], dqkv)
        lin_abs(f"{p}.in", hin, dqkv)
        dh = add(ds1, dhin_attn)
    newP, newV = dict(P), {}
    for n in sorted(g):
        newP[n], newV[n] = sgd(P[n], g[n], V.get(n), lr, momentum, first)
    return loss, newP, newV, g
