"""Op-stream builders for the paper's client workloads (BASELINE.json configs):
toy MLP (config 1), ResNet-50 inference (config 2 HP) and MobileNetV2 training (config 2 BE).

A workload is a static list of liborion operators (R15: the unique kernel ID is the op's position
in the list) over device buffers that torch allocates once (PyTorch is only the allocator here;
every op runs in liborion's kernels). Layouts: activations NHWC fp32, conv weights OHWI, linear
[out, in], parameters/gradients/momentum in flat buffers so SGD is one launch.

The builders are independent of oracle/model.py (they define the same TorchVision architectures
separately; tests compare parameter specs and outputs).
"""
import math

import torch

from . import _lib as L
from .runtime import make_op, f32bits

F32 = torch.float32
EPS_BITS = f32bits(1e-5)


class Graph:
    """A client's op list plus the device buffers it references."""

    def __init__(self, name, device="cuda"):
        self.name = name
        self.device = device
        self.ops = []          # (fn_name or kind, args, label)
        self.bufs = {}
        self.ws_bytes = L.WS_TICKET_BYTES + 256
        self._ws = None
        self._ws_ops = []      # (op index, arg index of ws ptr, arg index of ws bytes)

    # ---- buffers
    def buf(self, name, shape, dtype=F32, zero=True):
        """A named device buffer. Asking again for an existing name returns the same tensor (the op
        lists hold raw pointers, so a buffer must never be replaced while the graph lives)."""
        old = self.bufs.get(name)
        if old is not None:
            assert tuple(old.shape) == tuple(shape) and old.dtype == dtype, f"buffer {name} redefined"
            return old
        t = torch.zeros(shape, dtype=dtype, device=self.device) if zero else torch.empty(shape, dtype=dtype, device=self.device)
        self.bufs[name] = t
        return t

    def need_ws(self, nbytes):
        self.ws_bytes = max(self.ws_bytes, int(nbytes))

    # ---- ops
    def k(self, fn, args, label, ws_at=None):
        self.ops.append((fn, list(args), label))
        if ws_at is not None:
            self._ws_ops.append((len(self.ops) - 1, ws_at))
        return len(self.ops) - 1

    def memcpy(self, kind, dst, src, nbytes, label):
        self.ops.append((kind, [dst, src, nbytes], label))

    def finalize(self):
        """Allocate the shared split/reduction workspace once per graph (ops of one client run in
        stream order, and every kernel leaves its tickets zeroed, so one workspace serves all ops and
        all variants) and patch its pointer into the ops that use it."""
        if self._ws is None or self._ws.numel() * 4 < self.ws_bytes:
            assert self._ws is None, "workspace grew after ops were patched"
            self._ws = torch.zeros(self.ws_bytes // 4 + 64, dtype=F32, device=self.device)
        for i, at in self._ws_ops:
            self.ops[i][1][at] = self._ws.data_ptr()
            self.ops[i][1][at + 1] = self.ws_bytes
        return self

    def orion_ops(self, profiles=None, kid_base=0):
        """liborion op records; profiles: {kernel_id: (cls, sm_needed, dur_ns)} (offline profile)."""
        out = []
        for i, (fn, args, label) in enumerate(self.ops):
            kid = kid_base + i
            cls, sm, dur = (profiles or {}).get(kid, (L.CLS_U, 0, 0))
            if isinstance(fn, str):
                out.append(make_op(fn, args, kernel_id=kid, cls=cls, sm_needed=sm, dur_ns=dur))
            else:
                out.append(make_op(0, args, kernel_id=kid, kind=fn))
        return out

    def labels(self):
        return [lab for _, _, lab in self.ops]

    def kernel_ops(self):
        return [(i, fn, args, lab) for i, (fn, args, lab) in enumerate(self.ops) if isinstance(fn, str)]


def _p(t):
    return t.data_ptr()


# ------------------------------------------------------------------------ generic layer helpers
def gemm(g, A, B, C, bias, M, N, K, lda, ldb, ldc, flags, label):
    ws = L.lib.orion_gemm_workspace_bytes(M, N, K) if not (M <= 8 and flags == 2) else 0
    args = [_p(A), _p(B), _p(C), _p(bias) if bias is not None else 0, M, N, K, lda, ldb, ldc, flags, 0, 0]
    if ws:
        g.need_ws(ws)
        return g.k("gemm", args, label, ws_at=11)
    return g.k("gemm", args, label)


def linear_fwd(g, x, w, b, y, label):
    """y[B, out] = x[B, in] W^T + b (flags = B^T)."""
    Bn, fin = x.shape
    fout = w.shape[0]
    return gemm(g, x, w, y, b, Bn, fout, fin, fin, fin, fout, 2, label)


def conv_args(x, w, y, stride, pad):
    n, h, wd, c = x.shape
    k, r, s, _ = w.shape
    p, q = y.shape[1], y.shape[2]
    return [n, h, wd, c, k, r, s, stride, pad, p, q]


def conv_fwd(g, x, w, y, stride, pad, label, depthwise=False):
    n, h, wd, c = x.shape
    k, r, s, cg = w.shape
    if depthwise:
        return g.k("dw_fwd", [_p(x), _p(w), _p(y)] + conv_args(x, w, y, stride, pad), label)
    if r == 1 and s == 1 and stride == 1 and pad == 0:   # 1x1 conv = GEMM [NHW, C] x [K, C]^T
        return gemm(g, x, w, y, None, n * h * wd, k, c, c, c, k, 2, label)
    p_, q_ = y.shape[1], y.shape[2]
    g.need_ws(L.lib.orion_gemm_workspace_bytes(n * p_ * q_, k, r * s * c))
    return g.k("conv_fwd", [_p(x), _p(w), _p(y)] + conv_args(x, w, y, stride, pad) + [0, 0], label, ws_at=14)


def conv_dgrad(g, dy, w, dx, stride, pad, label, depthwise=False):
    n, h, wd, c = dx.shape
    k, r, s, _ = w.shape
    if depthwise:
        return g.k("dw_dgrad", [_p(dy), _p(w), _p(dx)] + conv_args(dx, w, dy, stride, pad), label)
    if r == 1 and s == 1 and stride == 1 and pad == 0:   # dx[NHW, C] = dy[NHW, K] W[K, C]
        return gemm(g, dy, w, dx, None, n * h * wd, c, k, k, c, c, 0, label)
    if c % 4 == 0:
        # col[NPQ, RSC] = dy[NPQ, K] W[K, RSC] (dense streaming GEMM: no zero taps, K-major loads),
        # then dx = col2im(col); measured 3-10x faster than the implicit-GEMM data gradient
        # (per-element tap decode) at ResNet-50's batch-64 shapes
        p_, q_ = dy.shape[1], dy.shape[2]
        col = g.buf(f"col.{label}", (n * p_ * q_, r * s * c))
        gemm(g, dy, w, col, None, n * p_ * q_, r * s * c, k, k, r * s * c, r * s * c, 0, f"{label}.col")
        return g.k("col2im", [_p(col), _p(dx), n, h, wd, c, r, s, stride, pad, p_, q_], label)
    g.need_ws(L.lib.orion_gemm_workspace_bytes(n * h * wd, c, r * s * k))
    return g.k("conv_dgrad", [_p(dy), _p(w), _p(dx)] + conv_args(dx, w, dy, stride, pad) + [0, 0], label, ws_at=14)


def conv_wgrad(g, x, dy, dw, stride, pad, label, depthwise=False):
    n, h, wd, c = x.shape
    k, r, s, _ = dw.shape
    p, q = dy.shape[1], dy.shape[2]
    if depthwise:
        g.need_ws(L.lib.orion_dw_wgrad_workspace_bytes(n, c, p, q))
        return g.k("dw_wgrad", [_p(x), _p(dy), _p(dw)] + conv_args(x, dw, dy, stride, pad) + [0, 0], label, ws_at=14)
    if r == 1 and s == 1 and stride == 1 and pad == 0:   # dW[K, C] = dy^T[K, NHW] x[NHW, C]
        return gemm(g, dy, x, dw, None, k, c, n * h * wd, k, c, c, 1, label)
    g.need_ws(L.lib.orion_conv_wgrad_workspace_bytes(n, h, wd, c, k, r, s, stride, pad))
    return g.k("conv_wgrad", [_p(x), _p(dy), _p(dw)] + conv_args(x, dw, dy, stride, pad) + [0, 0], label, ws_at=14)


# ============================================================================ toy MLP (config 1)
def mlp_spec(width=512, layers=3):
    spec = []
    for i in range(layers):
        spec.append((f"fc{i}.w", (width, width), ("uniform_fan_in", width)))
        spec.append((f"fc{i}.b", (width,), ("uniform_fan_in", width)))
    return spec


class FlatParams:
    """Parameters (and their gradients / momentum) as views of flat device buffers."""

    def __init__(self, g, spec, host_params, trainable=None, grads=True, momentum=False):
        names = [n for n, _, _ in spec if trainable is None or n in trainable]
        self.spec = {n: s for n, s, _ in spec}
        total = sum(math.prod(self.spec[n]) for n in names)
        self.flat = g.buf("params.flat", (max(total, 1),))
        self.gflat = g.buf("grads.flat", (max(total, 1),)) if grads else None
        self.vflat = g.buf("momentum.flat", (max(total, 1),)) if momentum else None
        self.total = total
        self.p, self.g = {}, {}
        off = 0
        for n in names:
            sz = math.prod(self.spec[n])
            self.p[n] = self.flat[off:off + sz].view(self.spec[n])
            if grads:
                self.g[n] = self.gflat[off:off + sz].view(self.spec[n])
            off += sz
        for n, s, _ in spec:         # non-trainable tensors (BN running stats)
            if n not in self.p:
                self.p[n] = g.buf(n, s)
        self.host = host_params
        self.reset()

    def reset(self):
        """Restore the initial parameters / running stats and zero gradients and momentum."""
        with torch.no_grad():
            for n in self.p:
                self.p[n].copy_(self.host[n].to(self.p[n].device))
            if self.gflat is not None:
                self.gflat.zero_()
            if self.vflat is not None:
                self.vflat.zero_()


def mlp_infer_graph(host_params, batch=1, width=512, layers=3, device="cuda"):
    """HP: Linear-ReLU-Linear-ReLU-Linear inference with H2D input and D2H output memops."""
    g = Graph("mlp_infer", device)
    P = FlatParams(g, mlp_spec(width, layers), host_params, grads=False)
    x = g.buf("x", (batch, width))
    g.memcpy(L.OP_MEMCPY_H2D, _p(x), 0, x.numel() * 4, "h2d_input")
    h = x
    for i in range(layers):
        z = g.buf(f"z{i}", (batch, width))
        linear_fwd(g, h, P.p[f"fc{i}.w"], P.p[f"fc{i}.b"], z, f"fc{i}")
        h = z
        if i < layers - 1:
            a = g.buf(f"a{i}", (batch, width))
            g.k("relu", [_p(z), _p(a), z.numel()], f"relu{i}")
            h = a
    g.out = h
    g.memcpy(L.OP_MEMCPY_D2H, 0, _p(h), h.numel() * 4, "d2h_output")
    g.params = P
    return g.finalize()


def mlp_train_graph(host_params, xs, ts, lr=0.01, width=512, layers=3, device="cuda"):
    """BE: MLP training step (MSE loss, SGD momentum 0), one op-list variant per pre-staged batch.
    Returns (graph, variants) where variants[i] are the op lists for batch i."""
    g = Graph("mlp_train", device)
    P = FlatParams(g, mlp_spec(width, layers), host_params, grads=True, momentum=False)
    batch = xs[0].shape[0]
    xb = [g.buf(f"x{i}", tuple(x.shape)) for i, x in enumerate(xs)]
    tb = [g.buf(f"t{i}", tuple(t.shape)) for i, t in enumerate(ts)]
    with torch.no_grad():
        for d, s in zip(xb + tb, list(xs) + list(ts)):
            d.copy_(s.to(d.device))
    loss = g.buf("loss", (1,))
    z = [g.buf(f"z{i}", (batch, width)) for i in range(layers)]
    a = [g.buf(f"a{i}", (batch, width)) for i in range(layers - 1)]
    dz = [g.buf(f"dz{i}", (batch, width)) for i in range(layers)]
    da = [g.buf(f"da{i}", (batch, width)) for i in range(layers - 1)]
    g.need_ws(L.WS_TICKET_BYTES + 8 * 148 * 8)
    variants = []
    for vi in range(len(xs)):
        g.ops = []
        g._ws_ops = []
        x, t = xb[vi], tb[vi]
        h = x
        for i in range(layers):
            linear_fwd(g, h, P.p[f"fc{i}.w"], P.p[f"fc{i}.b"], z[i], f"fc{i}")
            h = z[i]
            if i < layers - 1:
                g.k("relu", [_p(z[i]), _p(a[i]), z[i].numel()], f"relu{i}")
                h = a[i]
        g.k("mse", [_p(z[-1]), _p(t), _p(loss), _p(dz[-1]), z[-1].numel(), 0, 0], "mse", ws_at=5)
        for i in reversed(range(layers)):
            inp = x if i == 0 else a[i - 1]
            w = P.p[f"fc{i}.w"]
            # dW = dz^T inp ; db = colsum(dz) ; d(inp) = dz W
            gemm(g, dz[i], inp, P.g[f"fc{i}.w"], None, width, width, batch, width, width, width, 1, f"fc{i}.wgrad")
            g.k("colsum", [_p(dz[i]), _p(P.g[f"fc{i}.b"]), batch, width], f"fc{i}.bgrad")
            if i > 0:
                gemm(g, dz[i], w, da[i - 1], None, batch, width, width, width, width, width, 0, f"fc{i}.dgrad")
                g.k("relu_bwd", [_p(z[i - 1]), _p(da[i - 1]), _p(dz[i - 1]), z[i - 1].numel()], f"relu{i - 1}.bwd")
        g.k("sgd", [_p(P.flat), _p(P.gflat), 0, P.total, f32bits(lr), f32bits(0.0)], "sgd")
        variants.append((g.ops, g._ws_ops))
    g.variants = []
    for ops, wso in variants:
        g.ops, g._ws_ops = ops, wso
        g.finalize()
        g.variants.append(list(g.ops))
    g.ops = g.variants[0]
    g.loss = loss
    g.params = P
    return g


# ====================================================================== ResNet-50 inference (HP)
RESNET50_LAYERS = [(64, 3, 1), (128, 4, 2), (256, 6, 2), (512, 3, 2)]
RESNET101_LAYERS = [(64, 3, 1), (128, 4, 2), (256, 23, 2), (512, 3, 2)]


def resnet_spec(layers=RESNET50_LAYERS, num_classes=1000):
    def bn(name, c):
        return [(f"{name}.gamma", (c,), ("const", 1.0)), (f"{name}.beta", (c,), ("const", 0.0)),
                (f"{name}.rmean", (c,), ("normal", 0.1)), (f"{name}.rvar", (c,), ("uniform", 0.5, 1.5))]

    def conv(name, cout, k, cin):
        return [(f"{name}.w", (cout, k, k, cin), ("kaiming_fan_out", cout * k * k))]
    s = conv("conv1", 64, 7, 3) + bn("bn1", 64)
    cin = 64
    for li, (w, nb, stride) in enumerate(layers):
        for bi in range(nb):
            p = f"layer{li + 1}.{bi}"
            s += conv(f"{p}.conv1", w, 1, cin) + bn(f"{p}.bn1", w)
            s += conv(f"{p}.conv2", w, 3, w) + bn(f"{p}.bn2", w)
            s += conv(f"{p}.conv3", 4 * w, 1, w) + bn(f"{p}.bn3", 4 * w)
            if bi == 0:
                s += conv(f"{p}.down", 4 * w, 1, cin) + bn(f"{p}.downbn", 4 * w)
            cin = 4 * w
    s += [("fc.w", (num_classes, cin), ("uniform_fan_in", cin)), ("fc.b", (num_classes,), ("uniform_fan_in", cin))]
    return s


def resnet_infer_graph(host_params, batch=4, hw=224, layers=RESNET50_LAYERS, num_classes=1000, device="cuda"):
    """HP: TorchVision ResNet v1.5 inference, eval BN, unfused ops (conv, BN, ReLU, add each a kernel,
    as PyTorch eager dispatches them: P:888-899), H2D input and D2H logits."""
    g = Graph("resnet_infer", device)
    spec = resnet_spec(layers, num_classes)
    P = FlatParams(g, spec, host_params, grads=False)
    x = g.buf("x", (batch, hw, hw, 3))
    g.memcpy(L.OP_MEMCPY_H2D, _p(x), 0, x.numel() * 4, "h2d_input")
    cnt = [0]

    def new(shape):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", shape)

    def cbr(h, name, bn, stride, pad, act=True):
        w = P.p[f"{name}.w"]
        n, hh, ww, _ = h.shape
        k = w.shape[1]
        ho, wo = (hh + 2 * pad - k) // stride + 1, (ww + 2 * pad - k) // stride + 1
        z = new((n, ho, wo, w.shape[0]))
        conv_fwd(g, h, w, z, stride, pad, name)
        y = new(z.shape)
        g.k("bn_eval", [_p(z), _p(y), _p(P.p[f"{bn}.gamma"]), _p(P.p[f"{bn}.beta"]), _p(P.p[f"{bn}.rmean"]),
                        _p(P.p[f"{bn}.rvar"]), n * ho * wo, w.shape[0], EPS_BITS], bn)
        if not act:
            return y
        a = new(y.shape)
        g.k("relu", [_p(y), _p(a), y.numel()], f"{bn}.relu")
        return a

    h = cbr(x, "conv1", "bn1", 2, 3)
    n, hh, ww, c = h.shape
    pq = (hh + 2 - 3) // 2 + 1
    m = new((n, pq, pq, c))
    g.k("maxpool", [_p(h), _p(m), n, hh, ww, c, pq, pq], "maxpool")
    h = m
    for li, (w, nb, stride) in enumerate(layers):
        for bi in range(nb):
            p = f"layer{li + 1}.{bi}"
            s = stride if bi == 0 else 1
            o = cbr(h, f"{p}.conv1", f"{p}.bn1", 1, 0)
            o = cbr(o, f"{p}.conv2", f"{p}.bn2", s, 1)
            o = cbr(o, f"{p}.conv3", f"{p}.bn3", 1, 0, act=False)
            idn = cbr(h, f"{p}.down", f"{p}.downbn", s, 0, act=False) if bi == 0 else h
            sm = new(o.shape)
            g.k("add", [_p(o), _p(idn), _p(sm), o.numel()], f"{p}.add")
            r = new(o.shape)
            g.k("relu", [_p(sm), _p(r), sm.numel()], f"{p}.relu")
            h = r
    n, hh, ww, c = h.shape
    pooled = new((n, c))
    g.k("avgpool", [_p(h), _p(pooled), n, hh * ww, c], "avgpool")
    logits = new((n, num_classes))
    linear_fwd(g, pooled, P.p["fc.w"], P.p["fc.b"], logits, "fc")
    g.memcpy(L.OP_MEMCPY_D2H, 0, _p(logits), logits.numel() * 4, "d2h_logits")
    g.out = logits
    g.x = x
    g.params = P
    return g.finalize()


# ================================================================= MobileNetV2 training (BE)
MNV2_SETTINGS = [(1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2), (6, 96, 3, 1), (6, 160, 3, 2), (6, 320, 1, 1)]


def mnv2_blocks():
    blocks, cin, i = [], 32, 1
    for t, c, n, s in MNV2_SETTINGS:
        for j in range(n):
            stride = s if j == 0 else 1
            blocks.append((f"features.{i}", cin, cin * t, c, stride, t != 1, stride == 1 and cin == c))
            cin = c
            i += 1
    return blocks


def mnv2_spec(num_classes=1000, eval_stats=False):
    """eval_stats: seeded running statistics (inference clients, R22) instead of torch's (0, 1) start."""
    def bn(name, c):
        st = [(f"{name}.rmean", (c,), ("normal", 0.1)), (f"{name}.rvar", (c,), ("uniform", 0.5, 1.5))] if eval_stats else \
             [(f"{name}.rmean", (c,), ("const", 0.0)), (f"{name}.rvar", (c,), ("const", 1.0))]
        return [(f"{name}.gamma", (c,), ("const", 1.0)), (f"{name}.beta", (c,), ("const", 0.0))] + st

    def conv(name, cout, k, cin):
        return [(f"{name}.w", (cout, k, k, cin), ("kaiming_fan_out", cout * k * k))]
    s = conv("features.0", 32, 3, 3) + bn("features.0.bn", 32)
    for name, cin, hid, cout, stride, expand, res in mnv2_blocks():
        if expand:
            s += conv(f"{name}.expand", hid, 1, cin) + bn(f"{name}.expand_bn", hid)
        s += conv(f"{name}.dw", hid, 3, 1) + bn(f"{name}.dw_bn", hid)
        s += conv(f"{name}.project", cout, 1, hid) + bn(f"{name}.project_bn", cout)
    s += conv("features.18", 1280, 1, 320) + bn("features.18.bn", 1280)
    s += [("classifier.w", (num_classes, 1280), ("normal", 0.01)), ("classifier.b", (num_classes,), ("const", 0.0))]
    return s


def mnv2_train_graph(host_params, xs, labels, lr=0.01, momentum=0.9, num_classes=1000, device="cuda"):
    """BE: one MobileNetV2 training iteration (train-mode BN, ReLU6, CE, SGD momentum), dropout p=0
    (reading R22). One op-list variant per pre-staged batch (8 batches cycled)."""
    g = Graph("mnv2_train", device)
    spec = mnv2_spec(num_classes)
    trainable = {n for n, _, _ in spec if not n.endswith((".rmean", ".rvar"))}
    P = FlatParams(g, spec, host_params, trainable=trainable, grads=True, momentum=True)
    batch, hw = xs[0].shape[0], xs[0].shape[1]
    xb = [g.buf(f"x{i}", tuple(x.shape)) for i, x in enumerate(xs)]
    lb = [g.buf(f"lab{i}", (batch,), dtype=torch.int32) for i in range(len(xs))]
    with torch.no_grad():
        for d, s in zip(xb, xs):
            d.copy_(s.to(d.device))
        for d, s in zip(lb, labels):
            d.copy_(s.to(d.device))
    loss = g.buf("loss", (1,))
    cnt = [0]

    def new(shape):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", shape)

    # ---- allocate activations / gradient buffers once (shared by all variants)
    layers = []   # (cname, bname, k, stride, depthwise, act, in_shape, out_shape)

    def plan(cname, bname, cin_shape, cout, k, stride, dw, act):
        n, h, w, c = cin_shape
        pad = k // 2
        ho, wo = (h + 2 * pad - k) // stride + 1, (w + 2 * pad - k) // stride + 1
        L_ = dict(cname=cname, bname=bname, k=k, stride=stride, pad=pad, dw=dw, act=act, cout=cout, in_shape=cin_shape,
                  z=new((n, ho, wo, cout)), y=new((n, ho, wo, cout)),
                  mean=new((cout,)), invstd=new((cout,)),
                  a=new((n, ho, wo, cout)) if act else None,
                  dy=new((n, ho, wo, cout)) if act else None, dz=new((n, ho, wo, cout)))
        layers.append(L_)
        return (n, ho, wo, cout)

    shape = plan("features.0", "features.0.bn", (batch, hw, hw, 3), 32, 3, 2, False, True)
    blocks = []
    for name, cin, hid, cout, stride, expand, res in mnv2_blocks():
        first = len(layers)
        in_shape = shape
        if expand:
            shape = plan(f"{name}.expand", f"{name}.expand_bn", shape, hid, 1, 1, False, True)
        shape = plan(f"{name}.dw", f"{name}.dw_bn", shape, hid, 3, stride, True, True)
        shape = plan(f"{name}.project", f"{name}.project_bn", shape, cout, 1, 1, False, False)
        blk = dict(first=first, last=len(layers) - 1, res=res, out=new(shape) if res else None,
                   in_shape=in_shape, dres=new(in_shape) if res else None)
        blocks.append(blk)
    shape = plan("features.18", "features.18.bn", shape, 1280, 1, 1, False, True)
    gin = [new(b["in_shape"]) for b in blocks] + [new(layers[-1]["in_shape"])]
    dtmp = {li: new(layers[li]["in_shape"]) for b in blocks for li in range(b["first"] + 1, b["last"] + 1)}
    n, hh, ww, c = shape
    pooled, logits, dlogits, dpooled, dfeat = new((n, c)), new((n, num_classes)), new((n, num_classes)), new((n, c)), new(shape)
    for L_ in layers:
        g.need_ws(L.lib.orion_bn_workspace_bytes(L_["z"].shape[0] * L_["z"].shape[1] * L_["z"].shape[2], L_["cout"]))
    g.need_ws(L.WS_TICKET_BYTES + 4 * batch)

    def conv_bn_fwd(L_, h):
        w = P.p[f"{L_['cname']}.w"]
        conv_fwd(g, h, w, L_["z"], L_["stride"], L_["pad"], L_["cname"], depthwise=L_["dw"])
        rows = L_["z"].numel() // L_["cout"]
        b = L_["bname"]
        g.k("bn_stats", [_p(L_["z"]), _p(L_["mean"]), _p(L_["invstd"]), _p(P.p[f"{b}.rmean"]), _p(P.p[f"{b}.rvar"]),
                         rows, L_["cout"], EPS_BITS, f32bits(0.1), 0, 0], f"{b}.stats", ws_at=9)
        g.k("bn_apply", [_p(L_["z"]), _p(L_["y"]), _p(P.p[f"{b}.gamma"]), _p(P.p[f"{b}.beta"]), _p(L_["mean"]),
                         _p(L_["invstd"]), rows, L_["cout"]], f"{b}.apply")
        L_["in"] = h
        if L_["act"]:
            g.k("relu6", [_p(L_["y"]), _p(L_["a"]), L_["y"].numel()], f"{b}.relu6")
            return L_["a"]
        return L_["y"]

    def conv_bn_bwd(L_, dout, dx):
        b = L_["bname"]
        rows = L_["z"].numel() // L_["cout"]
        dy = dout
        if L_["act"]:
            g.k("relu6_bwd", [_p(L_["y"]), _p(dout), _p(L_["dy"]), dout.numel()], f"{b}.relu6_bwd")
            dy = L_["dy"]
        g.k("bn_bwd_reduce", [_p(L_["z"]), _p(dy), _p(L_["mean"]), _p(L_["invstd"]), _p(P.g[f"{b}.gamma"]),
                              _p(P.g[f"{b}.beta"]), rows, L_["cout"], 0, 0], f"{b}.bwd_reduce", ws_at=8)
        g.k("bn_bwd_dx", [_p(L_["z"]), _p(dy), _p(L_["dz"]), _p(P.p[f"{b}.gamma"]), _p(L_["mean"]), _p(L_["invstd"]),
                          _p(P.g[f"{b}.gamma"]), _p(P.g[f"{b}.beta"]), rows, L_["cout"]], f"{b}.bwd_dx")
        w = P.p[f"{L_['cname']}.w"]
        conv_wgrad(g, L_["in"], L_["dz"], P.g[f"{L_['cname']}.w"], L_["stride"], L_["pad"], f"{L_['cname']}.wgrad",
                   depthwise=L_["dw"])
        if dx is not None:
            conv_dgrad(g, L_["dz"], w, dx, L_["stride"], L_["pad"], f"{L_['cname']}.dgrad", depthwise=L_["dw"])

    variants, ws_ops = [], None
    for vi in range(len(xs)):
        g.ops, g._ws_ops = [], []
        h = conv_bn_fwd(layers[0], xb[vi])
        for blk in blocks:
            inp = h
            for li in range(blk["first"], blk["last"] + 1):
                h = conv_bn_fwd(layers[li], h)
            if blk["res"]:
                g.k("add", [_p(h), _p(inp), _p(blk["out"]), h.numel()], f"block{blk['first']}.add")
                h = blk["out"]
        h = conv_bn_fwd(layers[-1], h)
        g.k("avgpool", [_p(h), _p(pooled), n, hh * ww, c], "avgpool")
        linear_fwd(g, pooled, P.p["classifier.w"], P.p["classifier.b"], logits, "classifier")
        g.k("ce", [_p(logits), _p(lb[vi]), _p(loss), _p(dlogits), n, num_classes, 0, 0], "ce", ws_at=6)
        gemm(g, dlogits, pooled, P.g["classifier.w"], None, num_classes, c, n, num_classes, c, c, 1, "classifier.wgrad")
        g.k("colsum", [_p(dlogits), _p(P.g["classifier.b"]), n, num_classes], "classifier.bgrad")
        gemm(g, dlogits, P.p["classifier.w"], dpooled, None, n, c, num_classes, num_classes, c, c, 0, "classifier.dgrad")
        g.k("avgpool_bwd", [_p(dpooled), _p(dfeat), n, hh * ww, c], "avgpool_bwd")
        # gin[b] = gradient w.r.t. the input of block b; gin[len(blocks)] = w.r.t. features.18's input
        conv_bn_bwd(layers[-1], dfeat, gin[len(blocks)])
        for bi in reversed(range(len(blocks))):
            blk = blocks[bi]
            dout = gin[bi + 1]
            dd = dout
            for li in range(blk["last"], blk["first"] - 1, -1):
                if li == blk["first"]:
                    out = blk["dres"] if blk["res"] else gin[bi]
                else:
                    out = dtmp[li]
                conv_bn_bwd(layers[li], dd, out)
                dd = out
            if blk["res"]:
                g.k("add", [_p(blk["dres"]), _p(dout), _p(gin[bi]), dout.numel()], f"block{bi}.add_bwd")
        d = gin[0]
        conv_bn_bwd(layers[0], d, None)
        g.k("sgd", [_p(P.flat), _p(P.gflat), _p(P.vflat), P.total, f32bits(lr), f32bits(momentum)], "sgd")
        variants.append(g.ops)
        ws_ops = g._ws_ops
    g.variants = []
    for ops in variants:
        g.ops, g._ws_ops = ops, list(ws_ops)
        g.finalize()
        g.variants.append(list(g.ops))
    g.ops = g.variants[0]
    g.loss = loss
    g.params = P
    g.logits = logits
    g.bn_out = {L_["bname"]: L_["y"] for L_ in layers}   # BN outputs (ReLU6 inputs), for parity tests
    return g


# ====================================================================== ResNet training (BE, config 3)
def resnet_train_spec(layers=RESNET50_LAYERS, num_classes=1000):
    """Training ResNet: BN running stats start at torch's defaults (mean 0, var 1)."""
    spec = []
    for n, s, init in resnet_spec(layers, num_classes):
        if n.endswith(".rmean"):
            init = ("const", 0.0)
        elif n.endswith(".rvar"):
            init = ("const", 1.0)
        spec.append((n, s, init))
    return spec


def resnet_train_graph(host_params, xs, labels, layers=RESNET50_LAYERS, lr=0.01, momentum=0.9, num_classes=1000,
                       device="cuda"):
    """BE (config 3): one TorchVision ResNet v1.5 training iteration — conv, train-mode BN, ReLU,
    residual add, max-pool, CE, SGD(momentum) — each op its own kernel, backward op by op in reverse
    order. One op-list variant per pre-staged batch."""
    g = Graph("resnet_train", device)
    spec = resnet_train_spec(layers, num_classes)
    trainable = {n for n, _, _ in spec if not n.endswith((".rmean", ".rvar"))}
    P = FlatParams(g, spec, host_params, trainable=trainable, grads=True, momentum=True)
    batch, hw = xs[0].shape[0], xs[0].shape[1]
    xb = [g.buf(f"x{i}", tuple(x.shape)) for i, x in enumerate(xs)]
    lb = [g.buf(f"lab{i}", (batch,), dtype=torch.int32) for i in range(len(xs))]
    with torch.no_grad():
        for d, s in zip(xb, xs):
            d.copy_(s.to(d.device))
        for d, s in zip(lb, labels):
            d.copy_(s.to(d.device))
    loss = g.buf("loss", (1,))
    cnt = [0]

    def new(shape):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", shape)

    def plan(cname, bname, in_shape, cout, k, stride, pad):
        n, h, w, _ = in_shape
        ho, wo = (h + 2 * pad - k) // stride + 1, (w + 2 * pad - k) // stride + 1
        L_ = dict(cname=cname, bname=bname, stride=stride, pad=pad, cout=cout, in_shape=in_shape,
                  z=new((n, ho, wo, cout)), y=new((n, ho, wo, cout)), mean=new((cout,)), invstd=new((cout,)),
                  dz=new((n, ho, wo, cout)))
        g.need_ws(L.lib.orion_bn_workspace_bytes(n * ho * wo, cout))
        return L_

    stem = plan("conv1", "bn1", (batch, hw, hw, 3), 64, 7, 2, 3)
    s_shape = stem["y"].shape
    a0, da0, dy0 = new(s_shape), new(s_shape), new(s_shape)
    n_, h_, w_, c_ = s_shape
    pq = (h_ + 2 - 3) // 2 + 1
    mp = new((n_, pq, pq, c_))
    shape = tuple(mp.shape)
    blocks = []
    cin = 64
    for li, (wd, nb, stride) in enumerate(layers):
        for bi in range(nb):
            p = f"layer{li + 1}.{bi}"
            s = stride if bi == 0 else 1
            b = dict(name=p, in_shape=shape)
            b["c1"] = plan(f"{p}.conv1", f"{p}.bn1", shape, wd, 1, 1, 0)
            b["a1"], b["d1"] = new(b["c1"]["y"].shape), new(b["c1"]["y"].shape)
            b["c2"] = plan(f"{p}.conv2", f"{p}.bn2", tuple(b["c1"]["y"].shape), wd, 3, s, 1)
            b["a2"], b["d2"] = new(b["c2"]["y"].shape), new(b["c2"]["y"].shape)
            b["c3"] = plan(f"{p}.conv3", f"{p}.bn3", tuple(b["c2"]["y"].shape), 4 * wd, 1, 1, 0)
            b["down"] = plan(f"{p}.down", f"{p}.downbn", shape, 4 * wd, 1, s, 0) if bi == 0 else None
            oshape = tuple(b["c3"]["y"].shape)
            b["sum"], b["out"], b["dsum"] = new(oshape), new(oshape), new(oshape)
            b["dmain"] = new(shape)
            b["din"] = new(shape)          # gradient w.r.t. the block input
            b["ddown"] = new(shape) if bi == 0 else None
            b["da2"], b["da1"] = new(b["c2"]["y"].shape), new(b["c1"]["y"].shape)
            blocks.append(b)
            shape = oshape
            cin = 4 * wd
    n, hh, ww, c = shape
    pooled, logits, dlogits, dpooled, dfeat = new((n, c)), new((n, num_classes)), new((n, num_classes)), new((n, c)), new(shape)
    dmp = blocks[0]["din"]
    g.need_ws(L.WS_TICKET_BYTES + 4 * batch)

    def conv_bn(L_, h):
        conv_fwd(g, h, P.p[f"{L_['cname']}.w"], L_["z"], L_["stride"], L_["pad"], L_["cname"])
        rows = L_["z"].numel() // L_["cout"]
        bn = L_["bname"]
        g.k("bn_stats", [_p(L_["z"]), _p(L_["mean"]), _p(L_["invstd"]), _p(P.p[f"{bn}.rmean"]), _p(P.p[f"{bn}.rvar"]),
                         rows, L_["cout"], EPS_BITS, f32bits(0.1), 0, 0], f"{bn}.stats", ws_at=9)
        g.k("bn_apply", [_p(L_["z"]), _p(L_["y"]), _p(P.p[f"{bn}.gamma"]), _p(P.p[f"{bn}.beta"]), _p(L_["mean"]),
                         _p(L_["invstd"]), rows, L_["cout"]], f"{bn}.apply")
        L_["in"] = h
        return L_["y"]

    def conv_bn_bwd(L_, dy, dx):
        bn = L_["bname"]
        rows = L_["z"].numel() // L_["cout"]
        g.k("bn_bwd_reduce", [_p(L_["z"]), _p(dy), _p(L_["mean"]), _p(L_["invstd"]), _p(P.g[f"{bn}.gamma"]),
                              _p(P.g[f"{bn}.beta"]), rows, L_["cout"], 0, 0], f"{bn}.bwd_reduce", ws_at=8)
        g.k("bn_bwd_dx", [_p(L_["z"]), _p(dy), _p(L_["dz"]), _p(P.p[f"{bn}.gamma"]), _p(L_["mean"]), _p(L_["invstd"]),
                          _p(P.g[f"{bn}.gamma"]), _p(P.g[f"{bn}.beta"]), rows, L_["cout"]], f"{bn}.bwd_dx")
        w = P.p[f"{L_['cname']}.w"]
        conv_wgrad(g, L_["in"], L_["dz"], P.g[f"{L_['cname']}.w"], L_["stride"], L_["pad"], f"{L_['cname']}.wgrad")
        if dx is not None:
            conv_dgrad(g, L_["dz"], w, dx, L_["stride"], L_["pad"], f"{L_['cname']}.dgrad")

    def relu(x, y, label):
        g.k("relu", [_p(x), _p(y), x.numel()], label)

    def relu_bwd(x, dy, dx, label):
        g.k("relu_bwd", [_p(x), _p(dy), _p(dx), x.numel()], label)

    def add(a, b, c, label):
        g.k("add", [_p(a), _p(b), _p(c), a.numel()], label)

    variants, ws_ops = [], None
    for vi in range(len(xs)):
        g.ops, g._ws_ops = [], []
        y0 = conv_bn(stem, xb[vi])
        relu(y0, a0, "bn1.relu")
        g.k("maxpool", [_p(a0), _p(mp), n_, h_, w_, c_, pq, pq], "maxpool")
        h = mp
        for b in blocks:
            p = b["name"]
            relu(conv_bn(b["c1"], h), b["a1"], f"{p}.bn1.relu")
            relu(conv_bn(b["c2"], b["a1"]), b["a2"], f"{p}.bn2.relu")
            y3 = conv_bn(b["c3"], b["a2"])
            idn = conv_bn(b["down"], h) if b["down"] is not None else h
            add(y3, idn, b["sum"], f"{p}.add")
            relu(b["sum"], b["out"], f"{p}.relu")
            h = b["out"]
        g.k("avgpool", [_p(h), _p(pooled), n, hh * ww, c], "avgpool")
        linear_fwd(g, pooled, P.p["fc.w"], P.p["fc.b"], logits, "fc")
        g.k("ce", [_p(logits), _p(lb[vi]), _p(loss), _p(dlogits), n, num_classes, 0, 0], "ce", ws_at=6)
        gemm(g, dlogits, pooled, P.g["fc.w"], None, num_classes, c, n, num_classes, c, c, 1, "fc.wgrad")
        g.k("colsum", [_p(dlogits), _p(P.g["fc.b"]), n, num_classes], "fc.bgrad")
        gemm(g, dlogits, P.p["fc.w"], dpooled, None, n, c, num_classes, num_classes, c, c, 0, "fc.dgrad")
        g.k("avgpool_bwd", [_p(dpooled), _p(dfeat), n, hh * ww, c], "avgpool_bwd")
        dout = dfeat
        for bi in reversed(range(len(blocks))):
            b = blocks[bi]
            p = b["name"]
            relu_bwd(b["sum"], dout, b["dsum"], f"{p}.relu_bwd")
            conv_bn_bwd(b["c3"], b["dsum"], b["da2"])
            relu_bwd(b["c2"]["y"], b["da2"], b["d2"], f"{p}.bn2.relu_bwd")
            conv_bn_bwd(b["c2"], b["d2"], b["da1"])
            relu_bwd(b["c1"]["y"], b["da1"], b["d1"], f"{p}.bn1.relu_bwd")
            conv_bn_bwd(b["c1"], b["d1"], b["dmain"])
            if b["down"] is not None:
                conv_bn_bwd(b["down"], b["dsum"], b["ddown"])
                add(b["dmain"], b["ddown"], b["din"], f"{p}.add_bwd")
            else:
                add(b["dmain"], b["dsum"], b["din"], f"{p}.add_bwd")
            dout = b["din"]
        g.k("maxpool_bwd", [_p(a0), _p(dmp), _p(da0), n_, h_, w_, c_, pq, pq], "maxpool_bwd")
        relu_bwd(y0, da0, dy0, "bn1.relu_bwd")
        conv_bn_bwd(stem, dy0, None)
        g.k("sgd", [_p(P.flat), _p(P.gflat), _p(P.vflat), P.total, f32bits(lr), f32bits(momentum)], "sgd")
        variants.append(g.ops)
        ws_ops = g._ws_ops
    g.variants = []
    for ops in variants:
        g.ops, g._ws_ops = ops, list(ws_ops)
        g.finalize()
        g.variants.append(list(g.ops))
    g.ops = g.variants[0]
    g.loss = loss
    g.params = P
    g.logits = logits
    # values the ReLU backward decides on (BN outputs and residual sums), for decision-aligned parity
    g.relu_in = {"bn1": stem["y"]}
    for b in blocks:
        g.relu_in[f"{b['name']}.bn1"] = b["c1"]["y"]
        g.relu_in[f"{b['name']}.bn2"] = b["c2"]["y"]
        g.relu_in[f"{b['name']}.sum"] = b["sum"]
    return g


# ========================================================================= BERT inference (HP, config 3)
BF16 = torch.bfloat16


def bert_spec(layers=12, hidden=768, heads=12, ffn=3072, vocab=30522, max_pos=512, types=2):
    """BERT-base parameters (HuggingFace BertModel without pooler), Linear weights [out, in].
    Synthetic init (reading R22): weights, embeddings and biases N(0, 0.02); LayerNorm gamma
    U[0.9, 1.1], beta N(0, 0.02)."""
    nrm = ("normal", 0.02)
    s = [("emb.word", (vocab, hidden), nrm), ("emb.pos", (max_pos, hidden), nrm), ("emb.type", (types, hidden), nrm),
         ("emb.ln.gamma", (hidden,), ("uniform", 0.9, 1.1)), ("emb.ln.beta", (hidden,), nrm)]
    for i in range(layers):
        p = f"layer{i}"
        for nm, o, k in (("q", hidden, hidden), ("k", hidden, hidden), ("v", hidden, hidden), ("o", hidden, hidden),
                         ("ffn1", ffn, hidden), ("ffn2", hidden, ffn)):
            s += [(f"{p}.{nm}.w", (o, k), nrm), (f"{p}.{nm}.b", (o,), nrm)]
        for ln in ("ln1", "ln2"):
            s += [(f"{p}.{ln}.gamma", (hidden,), ("uniform", 0.9, 1.1)), (f"{p}.{ln}.beta", (hidden,), nrm)]
    return s


class BF16Params:
    """Inference parameters cast to bfloat16 (model.to(torch.bfloat16)), one device tensor each."""

    def __init__(self, g, spec, host_params):
        self.host = host_params
        self.p = {n: g.buf(f"param.{n}", s, dtype=BF16) for n, s, _ in spec}
        self.reset()

    def reset(self):
        with torch.no_grad():
            for n, t in self.p.items():
                t.copy_(self.host[n].to(BF16).to(t.device))


def bert_infer_graph(host_params, batch=8, seq=128, layers=12, heads=12, hidden=768, ffn=3072, vocab=30522,
                     device="cuda"):
    """HP (config 3): BertModel forward in bf16, PyTorch-eager op granularity with the fused SDPA
    attention kernel: per layer q, k, v projections, attention, output projection, residual add,
    LayerNorm, FFN up, GELU, FFN down, residual add, LayerNorm (12 kernels). H2D of the token ids
    (int32) first, D2H of the last hidden state (bf16) last."""
    g = Graph("bert_infer", device)
    spec = bert_spec(layers, hidden, heads, ffn, vocab)
    P = BF16Params(g, spec, host_params)
    rows = batch * seq
    ids = g.buf("ids", (rows,), dtype=torch.int32)
    g.memcpy(L.OP_MEMCPY_H2D, _p(ids), 0, rows * 4, "h2d_ids")
    cnt = [0]

    def new(cols):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", (rows, cols), dtype=BF16)

    def lin(x, name, out, k):
        g.k("gemm_bf16", [_p(x), _p(P.p[f"{name}.w"]), _p(out), _p(P.p[f"{name}.b"]), rows, out.shape[1], k], name)

    def ln(x, y, name):
        g.k("layernorm", [_p(x), _p(y), _p(P.p[f"{name}.gamma"]), _p(P.p[f"{name}.beta"]), rows, hidden, f32bits(1e-12)], name)

    e = new(hidden)
    g.k("embed", [_p(ids), _p(P.p["emb.word"]), _p(P.p["emb.pos"]), _p(P.p["emb.type"]), _p(e), batch, seq, hidden, vocab],
        "embed")
    h = new(hidden)
    ln(e, h, "emb.ln")
    for i in range(layers):
        p = f"layer{i}"
        q, k, v, a, o, s1, h1 = (new(hidden) for _ in range(7))
        f, fg, f2, s2, h2 = new(ffn), new(ffn), new(hidden), new(hidden), new(hidden)
        lin(h, f"{p}.q", q, hidden)
        lin(h, f"{p}.k", k, hidden)
        lin(h, f"{p}.v", v, hidden)
        g.k("attention", [_p(q), _p(k), _p(v), _p(a), batch, seq, heads, hidden // heads, hidden], f"{p}.attn")
        lin(a, f"{p}.o", o, hidden)
        g.k("add_bf16", [_p(o), _p(h), _p(s1), rows * hidden], f"{p}.add1")
        ln(s1, h1, f"{p}.ln1")
        lin(h1, f"{p}.ffn1", f, hidden)
        g.k("gelu", [_p(f), _p(fg), rows * ffn], f"{p}.gelu")
        lin(fg, f"{p}.ffn2", f2, ffn)
        g.k("add_bf16", [_p(f2), _p(h1), _p(s2), rows * hidden], f"{p}.add2")
        ln(s2, h2, f"{p}.ln2")
        h = h2
    g.memcpy(L.OP_MEMCPY_D2H, 0, _p(h), rows * hidden * 2, "d2h_hidden")
    g.out = h
    g.x = ids
    g.params = P
    return g.finalize()


# ============================================================ Transformer encoder training (BE, config 4)
def encoder_spec(layers=6, d=512, ffn=2048):
    """torch.nn.TransformerEncoderLayer parameters (packed in-projection [3d, d]); torch's init
    reading: U(+-1/sqrt(fan_in)) weights, zero attention biases, LN (1, 0)."""
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


def encoder_train_graph(host_params, xs, ts, layers=6, d=512, heads=8, ffn=2048, lr=0.01, momentum=0.9, device="cuda"):
    """BE (config 4): one training iteration of a post-LN Transformer-encoder stack (fp32, MSE to a
    target, SGD momentum), op by op: packed in-projection GEMM, attention, out-projection, residual
    add, LayerNorm, FFN (ReLU), residual add, LayerNorm; backward in reverse with the two-op
    attention backward. One op-list variant per pre-staged (x, t) batch."""
    g = Graph("encoder_train", device)
    spec = encoder_spec(layers, d, ffn)
    P = FlatParams(g, spec, host_params, grads=True, momentum=True)
    b, sq, _ = xs[0].shape
    rows = b * sq
    xb = [g.buf(f"x{i}", (rows, d)) for i in range(len(xs))]
    tb = [g.buf(f"tgt{i}", (rows, d)) for i in range(len(ts))]
    with torch.no_grad():
        for dst, src in zip(xb + tb, list(xs) + list(ts)):
            dst.copy_(src.reshape(rows, d).to(dst.device))
    loss = g.buf("loss", (1,))
    cnt = [0]

    def new(cols):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", (rows, cols))
    L_ = []
    for i in range(layers):
        L_.append(dict(qkv=new(3 * d), a=new(d), o=new(d), s1=new(d), h1=new(d), m1=g.buf(f"m1_{i}", (rows,)),
                       r1=g.buf(f"r1_{i}", (rows,)), f=new(ffn), fa=new(ffn), f2=new(d), s2=new(d), h2=new(d),
                       m2=g.buf(f"m2_{i}", (rows,)), r2=g.buf(f"r2_{i}", (rows,))))
    dh, ds2, dfa, df, dh1ff, dh1, ds1, da, dqkv, dha = (new(c) for c in (d, d, ffn, ffn, d, d, d, d, 3 * d, d))
    dhs = [new(d) for _ in range(layers)]
    stats = g.buf("attn_stats", (b * heads * sq * 3,))
    g.need_ws(L.lib.orion_layernorm_bwd_workspace_bytes(rows, d))
    g.need_ws(L.WS_TICKET_BYTES + 8 * 148 * 8)
    eps = f32bits(1e-5)

    def lin(x, name, out):
        linear_fwd(g, x, P.p[f"{name}.w"], P.p[f"{name}.b"], out, name)

    def lin_bwd(x, name, dy, dx):
        w = P.p[f"{name}.w"]
        fout, fin = w.shape
        gemm(g, dy, x, P.g[f"{name}.w"], None, fout, fin, rows, fout, fin, fin, 1, f"{name}.wgrad")
        g.k("colsum", [_p(dy), _p(P.g[f"{name}.b"]), rows, fout], f"{name}.bgrad")
        if dx is not None:
            gemm(g, dy, w, dx, None, rows, fin, fout, fout, fin, fin, 0, f"{name}.dgrad")

    def ln_bwd(x, dy, dx, name, m, r):
        g.k("layernorm_f32_bwd", [_p(x), _p(dy), _p(dx), _p(P.p[f"{name}.gamma"]), _p(m), _p(r), _p(P.g[f"{name}.gamma"]),
                                  _p(P.g[f"{name}.beta"]), rows, d, 0, 0], f"{name}.bwd", ws_at=10)

    variants, ws_ops = [], None
    for vi in range(len(xs)):
        g.ops, g._ws_ops = [], []
        h = xb[vi]
        for i in range(layers):
            p, R = f"enc{i}", L_[i]
            lin(h, f"{p}.in", R["qkv"])
            qkv = R["qkv"].data_ptr()
            g.k("attention_f32", [qkv, qkv + 4 * d, qkv + 8 * d, _p(R["a"]), b, sq, heads, d // heads, 3 * d, d], f"{p}.attn")
            lin(R["a"], f"{p}.out", R["o"])
            g.k("add", [_p(h), _p(R["o"]), _p(R["s1"]), rows * d], f"{p}.add1")
            g.k("layernorm_f32", [_p(R["s1"]), _p(R["h1"]), _p(P.p[f"{p}.ln1.gamma"]), _p(P.p[f"{p}.ln1.beta"]), _p(R["m1"]),
                                  _p(R["r1"]), rows, d, eps], f"{p}.ln1")
            lin(R["h1"], f"{p}.ff1", R["f"])
            g.k("relu", [_p(R["f"]), _p(R["fa"]), rows * ffn], f"{p}.relu")
            lin(R["fa"], f"{p}.ff2", R["f2"])
            g.k("add", [_p(R["h1"]), _p(R["f2"]), _p(R["s2"]), rows * d], f"{p}.add2")
            g.k("layernorm_f32", [_p(R["s2"]), _p(R["h2"]), _p(P.p[f"{p}.ln2.gamma"]), _p(P.p[f"{p}.ln2.beta"]), _p(R["m2"]),
                                  _p(R["r2"]), rows, d, eps], f"{p}.ln2")
            R["in"] = h
            h = R["h2"]
        g.k("mse", [_p(h), _p(tb[vi]), _p(loss), _p(dh), rows * d, 0, 0], "mse", ws_at=5)
        dcur = dh
        for i in reversed(range(layers)):
            p, R = f"enc{i}", L_[i]
            ln_bwd(R["s2"], dcur, ds2, f"{p}.ln2", R["m2"], R["r2"])
            lin_bwd(R["fa"], f"{p}.ff2", ds2, dfa)
            g.k("relu_bwd", [_p(R["f"]), _p(dfa), _p(df), rows * ffn], f"{p}.relu_bwd")
            lin_bwd(R["h1"], f"{p}.ff1", df, dh1ff)
            g.k("add", [_p(ds2), _p(dh1ff), _p(dh1), rows * d], f"{p}.add2_bwd")
            ln_bwd(R["s1"], dh1, ds1, f"{p}.ln1", R["m1"], R["r1"])
            lin_bwd(R["a"], f"{p}.out", ds1, da)
            qkv, dq = R["qkv"].data_ptr(), dqkv.data_ptr()
            g.k("attention_f32_bwd_dq", [qkv, qkv + 4 * d, qkv + 8 * d, _p(da), dq, _p(stats), b, sq, heads, d // heads, 3 * d, d],
                f"{p}.attn_bwd_dq")
            g.k("attention_f32_bwd_dkv", [qkv, qkv + 4 * d, qkv + 8 * d, _p(da), _p(stats), dq + 4 * d, dq + 8 * d, b, sq, heads,
                                          d // heads, 3 * d, d], f"{p}.attn_bwd_dkv")
            lin_bwd(R["in"], f"{p}.in", dqkv, dha)
            g.k("add", [_p(ds1), _p(dha), _p(dhs[i]), rows * d], f"{p}.add1_bwd")
            dcur = dhs[i]
        g.k("sgd", [_p(P.flat), _p(P.gflat), _p(P.vflat), P.total, f32bits(lr), f32bits(momentum)], "sgd")
        variants.append(g.ops)
        ws_ops = g._ws_ops
    g.variants = []
    for ops in variants:
        g.ops, g._ws_ops = ops, list(ws_ops)
        g.finalize()
        g.variants.append(list(g.ops))
    g.ops = g.variants[0]
    g.loss = loss
    g.params = P
    g.relu_in = {f"enc{i}.ff1": L_[i]["f"] for i in range(layers)}
    return g


# ============================================================ inference clients of the inf-inf config
def mnv2_infer_graph(host_params, batch=4, hw=224, num_classes=1000, device="cuda"):
    """Inf-inf BE client (Table 1: MobileNetV2 inference b4): TorchVision MobileNetV2
    in eval mode, unfused ops (conv, BN, ReLU6, add each a kernel), H2D input and D2H logits."""
    g = Graph("mnv2_infer", device)
    spec = mnv2_spec(num_classes, eval_stats=True)
    P = FlatParams(g, spec, host_params, grads=False)
    x = g.buf("x", (batch, hw, hw, 3))
    g.memcpy(L.OP_MEMCPY_H2D, _p(x), 0, x.numel() * 4, "h2d_input")
    cnt = [0]

    def new(shape):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", shape)

    def cb(h, cname, bname, k, stride, dw, act):
        w = P.p[f"{cname}.w"]
        n, hh, ww, _ = h.shape
        pad = k // 2
        ho, wo = (hh + 2 * pad - k) // stride + 1, (ww + 2 * pad - k) // stride + 1
        cout = w.shape[0]
        z = new((n, ho, wo, cout))
        conv_fwd(g, h, w, z, stride, pad, cname, depthwise=dw)
        y = new(z.shape)
        g.k("bn_eval", [_p(z), _p(y), _p(P.p[f"{bname}.gamma"]), _p(P.p[f"{bname}.beta"]), _p(P.p[f"{bname}.rmean"]),
                        _p(P.p[f"{bname}.rvar"]), n * ho * wo, cout, EPS_BITS], bname)
        if not act:
            return y
        a = new(y.shape)
        g.k("relu6", [_p(y), _p(a), y.numel()], f"{bname}.relu6")
        return a

    h = cb(x, "features.0", "features.0.bn", 3, 2, False, True)
    for name, cin, hid, cout, stride, expand, res in mnv2_blocks():
        inp = h
        if expand:
            h = cb(h, f"{name}.expand", f"{name}.expand_bn", 1, 1, False, True)
        h = cb(h, f"{name}.dw", f"{name}.dw_bn", 3, stride, True, True)
        h = cb(h, f"{name}.project", f"{name}.project_bn", 1, 1, False, False)
        if res:
            r = new(h.shape)
            g.k("add", [_p(h), _p(inp), _p(r), h.numel()], f"{name}.add")
            h = r
    h = cb(h, "features.18", "features.18.bn", 1, 1, False, True)
    n, hh, ww, c = h.shape
    pooled = new((n, c))
    g.k("avgpool", [_p(h), _p(pooled), n, hh * ww, c], "avgpool")
    logits = new((n, num_classes))
    linear_fwd(g, pooled, P.p["classifier.w"], P.p["classifier.b"], logits, "classifier")
    g.memcpy(L.OP_MEMCPY_D2H, 0, _p(logits), logits.numel() * 4, "d2h_logits")
    g.out, g.x, g.params = logits, x, P
    return g.finalize()


def encoder_infer_graph(host_params, batch=4, seq=192, layers=6, d=512, heads=8, ffn=2048, device="cuda"):
    """Inf-inf BE client: the "Transformer" (reading R32: post-LN encoder, 6 x d512 / 8 heads /
    FFN 2048) inference at Table 1's batch 4, fp32, the forward op list of encoder_train_graph;
    H2D of the input embeddings first, D2H of the last layer's output last."""
    g = Graph("encoder_infer", device)
    spec = encoder_spec(layers, d, ffn)
    P = FlatParams(g, spec, host_params, grads=False)
    rows = batch * seq
    x = g.buf("x", (rows, d))
    g.memcpy(L.OP_MEMCPY_H2D, _p(x), 0, x.numel() * 4, "h2d_input")
    cnt = [0]

    def new(cols):
        cnt[0] += 1
        return g.buf(f"t{cnt[0]}", (rows, cols))
    eps = f32bits(1e-5)
    mrow, rrow = g.buf("ln_mean", (rows,)), g.buf("ln_rstd", (rows,))
    h = x
    for i in range(layers):
        p = f"enc{i}"
        qkv, a, o, s1, h1, f, fa, f2, s2, h2 = new(3 * d), new(d), new(d), new(d), new(d), new(ffn), new(ffn), new(d), new(d), new(d)
        linear_fwd(g, h, P.p[f"{p}.in.w"], P.p[f"{p}.in.b"], qkv, f"{p}.in")
        q = qkv.data_ptr()
        g.k("attention_f32", [q, q + 4 * d, q + 8 * d, _p(a), batch, seq, heads, d // heads, 3 * d, d], f"{p}.attn")
        linear_fwd(g, a, P.p[f"{p}.out.w"], P.p[f"{p}.out.b"], o, f"{p}.out")
        g.k("add", [_p(h), _p(o), _p(s1), rows * d], f"{p}.add1")
        g.k("layernorm_f32", [_p(s1), _p(h1), _p(P.p[f"{p}.ln1.gamma"]), _p(P.p[f"{p}.ln1.beta"]), _p(mrow), _p(rrow), rows, d, eps],
            f"{p}.ln1")
        linear_fwd(g, h1, P.p[f"{p}.ff1.w"], P.p[f"{p}.ff1.b"], f, f"{p}.ff1")
        g.k("relu", [_p(f), _p(fa), rows * ffn], f"{p}.relu")
        linear_fwd(g, fa, P.p[f"{p}.ff2.w"], P.p[f"{p}.ff2.b"], f2, f"{p}.ff2")
        g.k("add", [_p(h1), _p(f2), _p(s2), rows * d], f"{p}.add2")
        g.k("layernorm_f32", [_p(s2), _p(h2), _p(P.p[f"{p}.ln2.gamma"]), _p(P.p[f"{p}.ln2.beta"]), _p(mrow), _p(rrow), rows, d, eps],
            f"{p}.ln2")
        h = h2
    g.memcpy(L.OP_MEMCPY_D2H, 0, _p(h), h.numel() * 4, "d2h_output")
    g.out, g.x, g.params = h, x, P
    return g.finalize()


# ============================================================ training as the HP client (config 4)
def as_hp_training(graph, x_host, device="cuda"):
    """Wrap a one-variant training graph as an HP client op list: H2D of the iteration's input batch
    first, D2H of the loss last (the request boundaries, R2 / R19); each 'request' is one training
    iteration (throughput mode). Returns (ops list, input buffer)."""
    xbuf = graph.bufs["x0"]
    ops = [(L.OP_MEMCPY_H2D, [xbuf.data_ptr(), 0, xbuf.numel() * 4], "h2d_batch")] + list(graph.variants[0])
    ops.append((L.OP_MEMCPY_D2H, [0, graph.loss.data_ptr(), 4], "d2h_loss"))
    graph.ops = ops
    graph.variants = [ops]
    return graph
