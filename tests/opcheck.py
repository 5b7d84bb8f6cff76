"""Teacher-forced per-op parity (test infrastructure): after the GPU ran a client's op list, recompute
each op's output with the fp64 oracle op (oracle/model.py) from the GPU's own input buffers and
compare. Works at full size because each op is checked on its own; buffers that later ops
overwrite in place (parameters after SGD, BN running stats) are checked against snapshots."""
import torch

from oracle import model as om
from paper_conf_eurosys_stratimk24_b200 import _lib as L


def _u2f(v):
    import struct
    return struct.unpack("<f", struct.pack("<I", v & 0xFFFFFFFF))[0]


class Resolver:
    """Map device pointers back to tensors (views) of a graph."""

    def __init__(self, tensors, read_alias=None):
        """read_alias: {real_tensor_ptr: snapshot tensor} — inputs read from a pre-run snapshot
        (parameters that SGD updates in place at the end of the iteration)."""
        self.items = []
        alias = read_alias or {}
        for t in tensors:
            if t is not None and t.numel():
                self.items.append((t.data_ptr(), t.data_ptr() + t.numel() * t.element_size(),
                                   alias.get(t.data_ptr(), t)))

    def get(self, ptr, numel, shape=None, dtype=torch.float32):
        for lo, hi, t in self.items:
            if lo <= ptr < hi and t.dtype == dtype:
                off = (ptr - lo) // t.element_size()
                flat = t.reshape(-1)
                v = flat[off:off + numel]
                return v.view(shape) if shape is not None else v
        raise KeyError(hex(ptr))


def rel(a, b, floor=1e-30):
    a, b = a.detach().double().cpu(), b.detach().double().cpu()
    return float((a - b).norm() / max(float(b.norm()), floor))


def check_op(fn, a, R, snap=None, R_in=None):
    """Return the relative error of op (fn, args a): outputs read through resolver R, inputs through
    R_in (defaults to R). snap: pre-op snapshots of tensors the op updates in place, by pointer."""
    snap = snap or {}
    R_in = R_in or R

    def T(ptr, numel, shape=None, dtype=torch.float32):
        if ptr in snap:
            return snap[ptr].reshape(-1)[:numel].view(shape) if shape is not None else snap[ptr].reshape(-1)[:numel]
        return R_in.get(ptr, numel, shape, dtype).cpu()
    if fn == "gemm":
        M, N, K, lda, ldb, ldc, fl = a[4], a[5], a[6], a[7], a[8], a[9], a[10]
        A = T(a[0], (K * lda) if fl & 1 else (M * lda)).view(K if fl & 1 else M, lda)
        B = T(a[1], (N * ldb) if fl & 2 else (K * ldb)).view(N if fl & 2 else K, ldb)
        Ad = A[:, :M].t() if fl & 1 else A[:, :K]
        Bd = B[:, :K].t() if fl & 2 else B[:, :N]
        ref = Ad.double() @ Bd.double()
        if a[3]:
            ref = ref + T(a[3], N).double()
        out = R.get(a[2], M * ldc).view(M, ldc)[:, :N]
        if fl & 1:
            # weight gradients reduce over N*H*W rows of mixed-sign terms: the error is normalised by
            # the absolute-term sum || |A|^T |B| || (a gradient is held to tol * max(1, kappa)
            # in rel L2, kappa = || |A|^T |B| || / || A^T B ||; the same as rel L2 when nothing cancels)
            absref = Ad.double().abs() @ Bd.double().abs()
            return rel(out, om._r(ref)) / max(1.0, float(absref.norm() / max(float(ref.norm()), 1e-30)))
        return rel(out, om._r(ref))
    if fn in ("conv_fwd", "conv_dgrad", "conv_wgrad", "dw_fwd", "dw_dgrad", "dw_wgrad"):
        n, h, w, c, k, r, s, st, pad, p, q = a[3:14]
        groups = c if fn.startswith("dw") else 1
        cg = 1 if groups > 1 else c
        if fn in ("conv_fwd", "dw_fwd"):
            x, wt = T(a[0], n * h * w * c, (n, h, w, c)), T(a[1], k * r * s * cg, (k, r, s, cg))
            return rel(R.get(a[2], n * p * q * k, (n, p, q, k)), om.conv2d_fwd(x, wt, st, pad, groups))
        if fn in ("conv_dgrad", "dw_dgrad"):
            dy, wt = T(a[0], n * p * q * k, (n, p, q, k)), T(a[1], k * r * s * cg, (k, r, s, cg))
            return rel(R.get(a[2], n * h * w * c, (n, h, w, c)), om.conv2d_bwd_data(dy, wt, (n, h, w, c), st, pad, groups))
        x, dy = T(a[0], n * h * w * c, (n, h, w, c)), T(a[1], n * p * q * k, (n, p, q, k))
        ref = om.conv2d_bwd_weight(x, dy, (k, r, s, cg), st, pad, groups)
        absref = om.conv2d_bwd_weight_abs(x, dy, (k, r, s, cg), st, pad, groups)
        kappa = max(1.0, float(absref.double().norm() / max(float(ref.double().norm()), 1e-30)))   # (as for gemm flags & 1)
        return rel(R.get(a[2], k * r * s * cg, (k, r, s, cg)), ref) / kappa
    if fn in ("relu", "relu6"):
        x = T(a[0], a[2])
        return rel(R.get(a[1], a[2]), (om.relu if fn == "relu" else om.relu6)(x))
    if fn in ("relu_bwd", "relu6_bwd", "add"):
        x, y = T(a[0], a[3]), T(a[1], a[3])
        f = {"relu_bwd": om.relu_bwd, "relu6_bwd": om.relu6_bwd, "add": om.add}[fn]
        return rel(R.get(a[2], a[3]), f(x, y))
    if fn == "bn_eval":
        rows, C = a[6], a[7]
        x = T(a[0], rows * C, (rows, C))
        ref = om.bn_eval(x, T(a[2], C), T(a[3], C), T(a[4], C), T(a[5], C), _u2f(a[8]))
        return rel(R.get(a[1], rows * C, (rows, C)), ref)
    if fn == "bn_stats":
        rows, C = a[5], a[6]
        x = T(a[0], rows * C, (rows, C))
        rm0, rv0 = T(a[3], C), T(a[4], C)     # snapshots (pre-update) required
        _, mean, invstd, rm, rv = om.bn_train_fwd(x, torch.ones(C), torch.zeros(C), rm0, rv0, _u2f(a[7]), _u2f(a[8]))
        return max(rel(R.get(a[1], C), mean), rel(R.get(a[2], C), invstd), rel(R.get(a[3], C), rm), rel(R.get(a[4], C), rv))
    if fn == "bn_apply":
        rows, C = a[6], a[7]
        x = T(a[0], rows * C, (rows, C)).double()
        ref = (x - T(a[4], C).double()) * T(a[5], C).double() * T(a[2], C).double() + T(a[3], C).double()
        return rel(R.get(a[1], rows * C, (rows, C)), om._r(ref))
    if fn == "bn_bwd_reduce":
        rows, C = a[6], a[7]
        x, dy = T(a[0], rows * C, (rows, C)), T(a[1], rows * C, (rows, C))
        _, dg, db = om.bn_bwd(x, dy, torch.ones(C), T(a[2], C), T(a[3], C))
        return max(rel(R.get(a[4], C), dg, 1e-3), rel(R.get(a[5], C), db, 1e-3))
    if fn == "bn_bwd_dx":
        rows, C = a[8], a[9]
        x, dy = T(a[0], rows * C, (rows, C)), T(a[1], rows * C, (rows, C))
        mean, invstd, gamma = T(a[4], C), T(a[5], C), T(a[3], C)
        dgamma, dbeta = T(a[6], C), T(a[7], C)
        xh = (x.double() - mean.double()) * invstd.double()
        ref = gamma.double() * invstd.double() / rows * (rows * dy.double() - dbeta.double() - xh * dgamma.double())
        return rel(R.get(a[2], rows * C, (rows, C)), om._r(ref))
    if fn == "maxpool":
        n, h, w, c, p, q = a[2:8]
        return rel(R.get(a[1], n * p * q * c, (n, p, q, c)), om.maxpool3x3s2(T(a[0], n * h * w * c, (n, h, w, c))))
    if fn == "avgpool":
        n, hw, c = a[2:5]
        return rel(R.get(a[1], n * c, (n, c)), om.avgpool_fwd(T(a[0], n * hw * c, (n, hw, 1, c))))
    if fn == "avgpool_bwd":
        n, hw, c = a[2:5]
        return rel(R.get(a[1], n * hw * c, (n, hw, 1, c)), om.avgpool_bwd(T(a[0], n * c, (n, c)), (n, hw, 1, c)))
    if fn == "ce":
        B, Cn = a[4], a[5]
        z = T(a[0], B * Cn, (B, Cn))
        lab = R.get(a[1], B, None, torch.int32).cpu()
        loss, dz = om.ce_fwd_bwd(z, lab)
        return max(rel(R.get(a[2], 1), loss.reshape(1)), rel(R.get(a[3], B * Cn, (B, Cn)), dz))
    BF = torch.bfloat16
    if fn == "gemm_bf16":
        M, N, K = a[4], a[5], a[6]
        x, w = T(a[0], M * K, (M, K), BF), T(a[1], N * K, (N, K), BF)
        b = T(a[3], N, None, BF) if a[3] else torch.zeros(N, dtype=BF)
        return rel(R.get(a[2], M * N, (M, N), BF), om.linear_any(x, w, b))
    if fn == "attention":
        B, S, H, d, ld = a[4:9]
        q, k, v = (T(a[i], B * S * ld, (B, S, ld), BF)[:, :, :H * d] for i in range(3))
        return rel(R.get(a[3], B * S * ld, (B, S, ld), BF)[:, :, :H * d], om.attention(q, k, v, H))
    if fn == "layernorm":
        rows, C = a[4], a[5]
        x = T(a[0], rows * C, (rows, C), BF)
        ref = om.layernorm(x, T(a[2], C, None, BF), T(a[3], C, None, BF), eps=_u2f(a[6]))
        return rel(R.get(a[1], rows * C, (rows, C), BF), ref)
    if fn == "gelu":
        return rel(R.get(a[1], a[2], None, BF), om.gelu(T(a[0], a[2], None, BF)))
    if fn == "add_bf16":
        return rel(R.get(a[2], a[3], None, BF), om.add_any(T(a[0], a[3], None, BF), T(a[1], a[3], None, BF)))
    if fn == "embed":
        B, S, H, V = a[5:9]
        ids = R.get(a[0], B * S, (B, S), torch.int32).cpu()
        ref = om.bert_embed(ids, T(a[1], V * H, (V, H), BF), T(a[2], S * H, (S, H), BF), T(a[3], H, (1, H), BF))
        return rel(R.get(a[4], B * S * H, (B, S, H), BF), ref)
    if fn == "maxpool_bwd":
        n, h, w, c, p, q = a[3:9]
        x, dy = T(a[0], n * h * w * c, (n, h, w, c)), T(a[1], n * p * q * c, (n, p, q, c))
        return rel(R.get(a[2], n * h * w * c, (n, h, w, c)), om.maxpool3x3s2_bwd(x, dy))
    if fn == "col2im":
        n, h, w, c, r, s_, st, pad, p, q = a[2:12]
        col = T(a[0], n * p * q * r * s_ * c, (n * p * q, r * s_ * c))
        return rel(R.get(a[1], n * h * w * c, (n, h, w, c)), om.col2im(col, (n, h, w, c), r, s_, st, pad))
    if fn == "layernorm_f32":
        rows, C = a[6], a[7]
        y, m, r = om.layernorm_fwd(T(a[0], rows * C, (rows, C)), T(a[2], C), T(a[3], C), _u2f(a[8]))
        return max(rel(R.get(a[1], rows * C, (rows, C)), y), rel(R.get(a[4], rows), m, 1e-3), rel(R.get(a[5], rows), r))
    if fn == "layernorm_f32_bwd":
        rows, C = a[8], a[9]
        dx, dg, db = om.layernorm_bwd(T(a[0], rows * C, (rows, C)), T(a[1], rows * C, (rows, C)), T(a[3], C), T(a[4], rows), T(a[5], rows))
        return max(rel(R.get(a[2], rows * C, (rows, C)), dx), rel(R.get(a[6], C), dg, 1e-3), rel(R.get(a[7], C), db, 1e-3))
    if fn in ("attention_f32", "attention_f32_bwd_dq", "attention_f32_bwd_dkv"):
        np_ = {"attention_f32": 4, "attention_f32_bwd_dq": 6, "attention_f32_bwd_dkv": 7}[fn]
        B, S, H, d, ldi, ldo = a[np_:np_ + 6]
        hd = H * d

        def view(ptr, ld):   # [B, S, hd] view of rows of stride ld starting at ptr
            return R_in.get(ptr, (B * S - 1) * ld + hd, None).cpu().as_strided((B, S, hd), (S * ld, ld, 1))

        def out(ptr, ld):
            return R.get(ptr, (B * S - 1) * ld + hd, None).cpu().as_strided((B, S, hd), (S * ld, ld, 1))
        q, k, v = view(a[0], ldi), view(a[1], ldi), view(a[2], ldi)
        if fn == "attention_f32":
            return rel(out(a[3], ldo), om.mha_fwd(q, k, v, H))
        dq, dk, dv = om.mha_bwd(q, k, v, view(a[3], ldo), H)
        if fn == "attention_f32_bwd_dq":
            return rel(out(a[4], ldi), dq)
        return max(rel(out(a[5], ldi), dk), rel(out(a[6], ldi), dv))
    if fn == "mse":
        n = a[4]
        loss, dy = om.mse_fwd_bwd(T(a[0], n), T(a[1], n))
        return max(rel(R.get(a[2], 1), loss.reshape(1)), rel(R.get(a[3], n), dy))
    if fn == "colsum":
        M, N = a[2], a[3]
        return rel(R.get(a[1], N), om._r(T(a[0], M * N, (M, N)).double().sum(0)))
    return None
