"""Operator parity on the GPU for config 3's operators: the bf16 transformer kernels (tcgen05
Linear, fused attention, LayerNorm, GELU, residual add, embedding) and the fp32 max-pool backward,
each called through the C ABI (orion_kernel_launch) against the fp64 oracle op (oracle/model.py) on
seeded inputs spanning several tiles plus ragged tails.

Tolerances: a bf16 op's oracle rounds its fp64 result once to bf16, the GPU rounds
its fp32 result once; the two differ only where the fp32/fp64 difference straddles a rounding
boundary (one bf16 ulp, 2^-8 relative, on a small fraction of elements), so rel L2 <= 2e-3. The
attention kernel also rounds the softmax probabilities to bf16 before P V (flash-style): 4e-3.
maxpool_bwd moves fp32 values and adds at most 4 of them: 1e-6. Every op is also run twice and must
give identical bytes."""
import pytest
import torch

from oracle import model as om
from synth import inputs as si

pytestmark = pytest.mark.gpu
BF = torch.bfloat16

if torch.cuda.is_available():
    import paper_conf_eurosys_stratimk24_b200 as orion
    from paper_conf_eurosys_stratimk24_b200.runtime import f32bits


def rel(a, b):
    a, b = a.detach().double().cpu(), b.detach().double().cpu()
    return float((a - b).norm() / max(float(b.norm()), 1e-30))


def run(fn, args, twice=None):
    s = torch.cuda.current_stream().cuda_stream
    ptrs = [a.data_ptr() if isinstance(a, torch.Tensor) else a for a in args]
    orion.kernel_launch(fn, ptrs, s)
    torch.cuda.synchronize()
    if twice is not None:
        first = twice.clone()
        orion.kernel_launch(fn, ptrs, s)
        torch.cuda.synchronize()
        assert torch.equal(first, twice), f"{fn} not deterministic"


def bfn(shape, seed, scale=1.0):
    return (si.normal(shape, seed) * scale).to(BF)


@pytest.mark.parametrize("M,N,K", [(1024, 768, 768), (1024, 3072, 768), (1024, 768, 3072), (1024, 2304, 768),
                                   (200, 136, 72), (130, 70, 40), (8, 64, 64), (1, 24, 8), (4100, 1000, 520)],
                         ids=str)
def test_gemm_bf16(M, N, K):
    x, w, b = bfn((M, K), 21), bfn((N, K), 22, 0.05), bfn((N,), 23, 0.1)
    y = torch.zeros(M, N, dtype=BF, device="cuda")
    run("gemm_bf16", [x.cuda(), w.cuda(), y, b.cuda(), M, N, K], twice=y)
    assert rel(y, om.linear_any(x, w, b)) < 2e-3
    y0 = torch.zeros(M, N, dtype=BF, device="cuda")   # no bias
    run("gemm_bf16", [x.cuda(), w.cuda(), y0, 0, M, N, K])
    assert rel(y0, om.linear_any(x, w, torch.zeros(N, dtype=BF))) < 2e-3


def test_gemm_bf16_rejects_unaligned_k():
    x = torch.zeros(16, 12, dtype=BF, device="cuda")
    w = torch.zeros(16, 12, dtype=BF, device="cuda")
    y = torch.zeros(16, 16, dtype=BF, device="cuda")
    with pytest.raises(Exception):
        run("gemm_bf16", [x, w, y, 0, 16, 16, 12])


@pytest.mark.parametrize("B,S,heads,ldpad", [(8, 128, 12, 0), (2, 64, 3, 0), (1, 32, 2, 64), (3, 16, 1, 8)], ids=str)
def test_attention(B, S, heads, ldpad):
    ld = heads * 64 + ldpad
    q, k, v = (bfn((B, S, ld), s) for s in (31, 32, 33))
    o = torch.zeros(B, S, ld, dtype=BF, device="cuda")
    run("attention", [q.cuda(), k.cuda(), v.cuda(), o, B, S, heads, 64, ld], twice=o)
    H = heads * 64
    ref = om.attention(q[:, :, :H], k[:, :, :H], v[:, :, :H], heads)
    assert rel(o[:, :, :H], ref) < 4e-3
    if ldpad:   # padding columns untouched
        assert torch.count_nonzero(o[:, :, H:]) == 0


@pytest.mark.parametrize("rows,C", [(1024, 768), (37, 2048), (5, 8), (1001, 1024)], ids=str)
def test_layernorm(rows, C):
    x = bfn((rows, C), 41, 3.0) + torch.tensor(2.0, dtype=BF)
    gm, bt = (1 + 0.1 * si.normal((C,), 42)).to(BF), bfn((C,), 43, 0.1)
    y = torch.zeros(rows, C, dtype=BF, device="cuda")
    run("layernorm", [x.cuda(), y, gm.cuda(), bt.cuda(), rows, C, f32bits(1e-12)], twice=y)
    assert rel(y, om.layernorm(x, gm, bt, eps=1e-12)) < 2e-3


def test_gelu_add_embed():
    n = 8 * 1001
    x, z = bfn((n,), 51, 3.0), bfn((n,), 52)
    y = torch.zeros(n, dtype=BF, device="cuda")
    run("gelu", [x.cuda(), y, n], twice=y)
    assert rel(y, om.gelu(x)) < 2e-3
    c = torch.zeros(n, dtype=BF, device="cuda")
    run("add_bf16", [x.cuda(), z.cuda(), c, n], twice=c)
    assert rel(c, om.add_any(x, z)) < 2e-3
    B, S, H, V = 2, 128, 768, 1000
    ids = si.token_ids((B, S), V, si.HP_SEED)
    word, pos, typ = bfn((V, H), 53, 0.02), bfn((512, H), 54, 0.02), bfn((2, H), 55, 0.02)
    out = torch.zeros(B, S, H, dtype=BF, device="cuda")
    run("embed", [ids.cuda(), word.cuda(), pos.cuda(), typ.cuda(), out, B, S, H, V], twice=out)
    assert rel(out, om.bert_embed(ids, word, pos, typ)) < 2e-3


@pytest.mark.parametrize("n,h,w,c", [(2, 112, 112, 64), (2, 15, 13, 8), (1, 4, 4, 4)], ids=str)
def test_maxpool_bwd(n, h, w, c):
    p, q = (h - 1) // 2 + 1, (w - 1) // 2 + 1
    x, dy = si.normal((n, h, w, c), 61), si.normal((n, p, q, c), 62)
    dx = torch.full((n, h, w, c), float("nan"), device="cuda")
    run("maxpool_bwd", [x.cuda(), dy.cuda(), dx, n, h, w, c, p, q], twice=dx)
    assert rel(dx, om.maxpool3x3s2_bwd(x, dy)) < 1e-6
    # ties (ReLU zeros feed the pool in ResNet): first maximum in row-major order takes the gradient
    xt = torch.relu(x - 1.0)
    run("maxpool_bwd", [xt.cuda(), dy.cuda(), dx, n, h, w, c, p, q])
    assert rel(dx, om.maxpool3x3s2_bwd(xt, dy)) < 1e-6


@pytest.mark.parametrize("n,h,w,c,k,st,pad", [(2, 56, 56, 256, 1, 2, 0), (2, 14, 14, 64, 3, 2, 1), (1, 9, 8, 4, 7, 2, 3),
                                               (2, 13, 11, 8, 3, 2, 1)], ids=str)
def test_col2im(n, h, w, c, k, st, pad):
    """fp32 col2im (strided conv data gradient, second half): vs the oracle's fold, and the pair
    GEMM + col2im vs the oracle's conv data gradient."""
    p, q = (h + 2 * pad - k) // st + 1, (w + 2 * pad - k) // st + 1
    col = si.normal((n * p * q, k * k * c), 63)
    dx = torch.full((n, h, w, c), float("nan"), device="cuda")
    run("col2im", [col.cuda(), dx, n, h, w, c, k, k, st, pad, p, q], twice=dx)
    assert rel(dx, om.col2im(col, (n, h, w, c), k, k, st, pad)) < 1e-6
