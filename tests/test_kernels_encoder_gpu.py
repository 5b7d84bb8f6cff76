"""Operator parity on the GPU for config 4's fp32 encoder-training operators (LayerNorm forward /
backward, attention forward and its two backward ops), through the C ABI, against the fp64
oracle ops on seeded inputs (packed in-projection strides, ragged row counts). Tolerance: per-tensor
relative L2 <= 2e-5 (fp32 storage and accumulation vs fp64); run twice -> identical."""
import pytest
import torch

from oracle import model as om
from synth import inputs as si

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_eurosys_stratimk24_b200 as orion
    from paper_conf_eurosys_stratimk24_b200 import _lib as L
    from paper_conf_eurosys_stratimk24_b200.runtime import f32bits


def rel(a, b, floor=1e-30):
    a, b = a.detach().double().cpu(), b.detach().double().cpu()
    return float((a - b).norm() / max(float(b.norm()), floor))


def run(fn, args, twice=()):
    s = torch.cuda.current_stream().cuda_stream
    ptrs = [a.data_ptr() if isinstance(a, torch.Tensor) else a for a in args]
    orion.kernel_launch(fn, ptrs, s)
    torch.cuda.synchronize()
    firsts = [t.clone() for t in twice]
    if twice:
        orion.kernel_launch(fn, ptrs, s)
        torch.cuda.synchronize()
        for f, t in zip(firsts, twice):
            assert torch.equal(f, t), f"{fn} not deterministic"


@pytest.mark.parametrize("rows,C", [(1536, 512), (100, 128), (65, 384)], ids=str)
def test_layernorm_f32(rows, C):
    x = si.normal((rows, C), 91) * 2 + 0.3
    g, b = 1 + 0.1 * si.normal((C,), 92), 0.1 * si.normal((C,), 93)
    y, m, r = (torch.zeros(rows, C, device="cuda"), torch.zeros(rows, device="cuda"), torch.zeros(rows, device="cuda"))
    run("layernorm_f32", [x.cuda(), y, g.cuda(), b.cuda(), m, r, rows, C, f32bits(1e-5)], twice=(y, m, r))
    yr, mr, rr = om.layernorm_fwd(x, g, b)
    assert rel(y, yr) < 2e-5 and rel(m, mr) < 2e-5 and rel(r, rr) < 2e-5
    dy = si.normal((rows, C), 94)
    dx, dg, db = torch.zeros(rows, C, device="cuda"), torch.zeros(C, device="cuda"), torch.zeros(C, device="cuda")
    wsb = torch.zeros(L.lib.orion_layernorm_bwd_workspace_bytes(rows, C) // 4 + 64, device="cuda")
    run("layernorm_f32_bwd", [x.cuda(), dy.cuda(), dx, g.cuda(), m, r, dg, db, rows, C, wsb, wsb.numel() * 4], twice=(dx, dg, db))
    dxr, dgr, dbr = om.layernorm_bwd(x, dy, g, m.cpu(), r.cpu())
    assert rel(dx, dxr) < 2e-5 and rel(dg, dgr) < 2e-5 and rel(db, dbr) < 2e-5


@pytest.mark.parametrize("B,S,H", [(2, 192, 8), (1, 32, 1), (3, 64, 2)], ids=str)
def test_attention_f32_fwd_bwd(B, S, H):
    d = 64
    hd = H * d
    qkv = si.normal((B, S, 3 * hd), 95)
    do = si.normal((B, S, hd), 96)
    q, k, v = (qkv[:, :, j * hd:(j + 1) * hd] for j in range(3))
    qkv_d = qkv.cuda()
    base = qkv_d.data_ptr()
    o = torch.zeros(B, S, hd, device="cuda")
    run("attention_f32", [base, base + 4 * hd, base + 8 * hd, o, B, S, H, d, 3 * hd, hd], twice=(o,))
    assert rel(o, om.mha_fwd(q, k, v, H)) < 2e-5
    dqkv = torch.zeros(B, S, 3 * hd, device="cuda")
    stats = torch.zeros(B * H * S * 3, device="cuda")
    g = dqkv.data_ptr()
    run("attention_f32_bwd_dq", [base, base + 4 * hd, base + 8 * hd, do.cuda(), g, stats, B, S, H, d, 3 * hd, hd], twice=(dqkv,))
    run("attention_f32_bwd_dkv", [base, base + 4 * hd, base + 8 * hd, do.cuda(), stats, g + 4 * hd, g + 8 * hd, B, S, H, d, 3 * hd, hd],
        twice=(dqkv,))
    dq, dk, dv = om.mha_bwd(q, k, v, do, H)
    assert rel(dqkv[:, :, :hd], dq) < 2e-5
    assert rel(dqkv[:, :, hd:2 * hd], dk) < 2e-5
    assert rel(dqkv[:, :, 2 * hd:], dv) < 2e-5
