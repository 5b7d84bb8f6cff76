"""Pins for the config-3/4 parts of the model oracle (oracle/model.py): the bf16 BERT forward
(HP of BASELINE config 3), ResNet training (BE of config 3, HP of config 4) and max-pool
backward. Each is pinned against something other than itself: HuggingFace's BertModel and
TorchVision's ResNet in fp64 with autograd (the models the paper ran),
explicit loops on tiny inputs, closed forms and invariants."""
import math

import pytest
import torch

from oracle import model as om
from synth import inputs as si
from test_oracle_model import _to_tv, _rn_rename

D = torch.float64


def _rand(*shape, seed=0, dtype=torch.float32):
    g = torch.Generator().manual_seed(seed)
    return torch.randn(*shape, generator=g, dtype=dtype)


# ------------------------------------------------------------------------------ elementwise
def test_gelu_erf_scalar_loop():
    x = _rand(257, seed=1, dtype=D) * 3
    y = om.gelu(x, store=D)
    for i in range(x.numel()):
        xv = float(x[i])
        assert abs(float(y[i]) - 0.5 * xv * (1 + math.erf(xv / math.sqrt(2)))) < 1e-14
    # special cases: gelu(0) = 0, gelu(x) -> x for large x, -> 0 for very negative x
    s = om.gelu(torch.tensor([0.0, 10.0, -10.0], dtype=D), store=D)
    assert float(s[0]) == 0.0 and abs(float(s[1]) - 10.0) < 1e-12 and abs(float(s[2])) < 1e-12


def test_layernorm_closed_form():
    x = _rand(6, 96, seed=2, dtype=D) * 5 + 3
    y = om.layernorm(x, torch.ones(96, dtype=D), torch.zeros(96, dtype=D), store=D)
    torch.testing.assert_close(y.mean(-1), torch.zeros(6, dtype=D), atol=1e-12, rtol=0)
    torch.testing.assert_close(((y - y.mean(-1, keepdim=True)) ** 2).mean(-1), torch.ones(6, dtype=D), atol=1e-9, rtol=0)
    # affine part: gamma scales, beta shifts each column
    g, b = _rand(96, seed=3, dtype=D), _rand(96, seed=4, dtype=D)
    y2 = om.layernorm(x, g, b, store=D)
    torch.testing.assert_close(y2, y * g + b, atol=1e-12, rtol=0)
    # a constant row normalises to beta (var 0, eps keeps it finite)
    c = om.layernorm(torch.full((1, 96), 2.5, dtype=D), g, b, store=D)
    torch.testing.assert_close(c[0], b, atol=1e-12, rtol=0)


def test_bf16_storage_rounding():
    """The bf16 ops round their fp64 result once, to nearest even (8 significant bits)."""
    one = torch.ones(1, dtype=D)
    vals = torch.tensor([1 + 2 ** -9, 1 + 3 * 2 ** -9, 1 + 2 ** -8 + 2 ** -10], dtype=D)
    r = om.add_any(vals, 0 * one).double()
    assert [float(v) for v in r] == [1.0, 1 + 2 ** -7, 1 + 2 ** -7]


def test_embedding_definition():
    V, S, H = 11, 5, 8
    word, pos, typ = _rand(V, H, seed=5, dtype=D), _rand(7, H, seed=6, dtype=D), _rand(2, H, seed=7, dtype=D)
    ids = torch.tensor([[3, 0, 10, 3, 1], [9, 9, 2, 4, 0]], dtype=torch.int32)
    e = om.bert_embed(ids, word, pos, typ, store=D)
    for b in range(2):
        for s in range(S):
            torch.testing.assert_close(e[b, s], word[int(ids[b, s])] + pos[s] + typ[0], atol=1e-14, rtol=0)


def test_attention_loops():
    """Explicit loops of softmax(q.k / sqrt d) v per head on a tiny input."""
    B, S, heads, d = 2, 3, 2, 4
    q, k, v = (_rand(B, S, heads * d, seed=s, dtype=D) for s in (8, 9, 10))
    o = om.attention(q, k, v, heads, store=D)
    for b in range(B):
        for h in range(heads):
            cols = slice(h * d, (h + 1) * d)
            for i in range(S):
                sc = [float((q[b, i, cols] * k[b, j, cols]).sum()) / math.sqrt(d) for j in range(S)]
                mx = max(sc)
                w = [math.exp(x - mx) for x in sc]
                z = sum(w)
                ref = sum(w[j] / z * v[b, j, cols] for j in range(S))
                torch.testing.assert_close(o[b, i, cols], ref, atol=1e-13, rtol=0)
    # invariant: with v constant per column the output equals it (softmax rows sum to 1)
    vc = torch.ones(B, S, heads * d, dtype=D) * torch.arange(heads * d, dtype=D)
    torch.testing.assert_close(om.attention(q, k, vc, heads, store=D), vc, atol=1e-13, rtol=0)


# ----------------------------------------------------------------------------- BERT model
def _hf_bert(P, layers, hidden, heads, ffn, vocab, max_pos):
    tr = pytest.importorskip("transformers")
    cfg = tr.BertConfig(vocab_size=vocab, hidden_size=hidden, num_hidden_layers=layers, num_attention_heads=heads,
                        intermediate_size=ffn, max_position_embeddings=max_pos, type_vocab_size=2, hidden_act="gelu",
                        hidden_dropout_prob=0.0, attention_probs_dropout_prob=0.0, layer_norm_eps=1e-12)
    try:
        m = tr.BertModel(cfg, add_pooling_layer=False, attn_implementation="eager")
    except TypeError:
        cfg._attn_implementation = "eager"
        m = tr.BertModel(cfg, add_pooling_layer=False)
    m = m.double().eval()
    sd = m.state_dict()
    ren = {"emb.word": "embeddings.word_embeddings.weight", "emb.pos": "embeddings.position_embeddings.weight",
           "emb.type": "embeddings.token_type_embeddings.weight", "emb.ln.gamma": "embeddings.LayerNorm.weight",
           "emb.ln.beta": "embeddings.LayerNorm.bias"}
    sub = {"q": "attention.self.query", "k": "attention.self.key", "v": "attention.self.value",
           "o": "attention.output.dense", "ln1": "attention.output.LayerNorm", "ffn1": "intermediate.dense",
           "ffn2": "output.dense", "ln2": "output.LayerNorm"}
    for k, v in P.items():
        if k in ren:
            tk = ren[k]
        else:
            li, part, leaf = k.split(".")
            tk = f"encoder.layer.{li[5:]}.{sub[part]}." + {"w": "weight", "b": "bias", "gamma": "weight", "beta": "bias"}[leaf]
        assert sd[tk].shape == v.shape, (k, tk)
        sd[tk] = v.double()
    m.load_state_dict(sd)
    return m


def test_bert_vs_huggingface_fp64():
    """The oracle's BERT, run unrounded (store = fp64), equals HuggingFace BertModel (eager
    attention, fp64) on a 2-layer model: pins every op's definition and the layer wiring."""
    L_, H, nh, F_, V, MP = 2, 64, 4, 128, 97, 40
    P = si.make_params(om.bert_spec(layers=L_, hidden=H, heads=nh, ffn=F_, vocab=V, max_pos=MP))
    Pd = om.to_model_dtype(P, D)
    ids = si.token_ids((3, 17), V, si.HP_SEED)
    y = om.bert_infer(Pd, ids, layers=L_, heads=nh, store=D)
    m = _hf_bert(P, L_, H, nh, F_, V, MP)
    with torch.no_grad():
        ref = m(input_ids=ids.long()).last_hidden_state
    assert float((y - ref).norm() / ref.norm()) < 1e-12


def test_bert_bf16_close_to_fp64():
    """bf16 storage with one rounding per op stays within the north_star's 2e-2 of the fp64
    model (a sanity bound on the accumulated rounding, not a tautology: a wrong rounding site,
    e.g. rounding inside the softmax, would not move it, but a dropped term would)."""
    L_, H, nh, F_, V, MP = 2, 128, 2, 256, 101, 64
    P = si.make_params(om.bert_spec(layers=L_, hidden=H, heads=nh, ffn=F_, vocab=V, max_pos=MP))
    ids = si.token_ids((2, 64), V, si.HP_SEED)
    yb = om.bert_infer(om.to_model_dtype(P), ids, layers=L_, heads=nh)
    yd = om.bert_infer(om.to_model_dtype(om.to_model_dtype(P), D), ids, layers=L_, heads=nh, store=D)
    assert yb.dtype == torch.bfloat16
    err = float((yb.double() - yd).norm() / yd.norm())
    assert 1e-4 < err < 2e-2, err


# -------------------------------------------------------------------------- max-pool backward
def test_maxpool_bwd_vs_autograd_and_loops():
    x = _rand(2, 9, 8, 3, seed=11)
    dy = _rand(2, 5, 4, 3, seed=12)
    dx = om.maxpool3x3s2_bwd(x, dy)
    xd = x.double().permute(0, 3, 1, 2).requires_grad_(True)
    y = torch.nn.functional.max_pool2d(xd, 3, 2, 1)
    y.backward(dy.double().permute(0, 3, 1, 2))
    torch.testing.assert_close(dx.double(), xd.grad.permute(0, 2, 3, 1), atol=1e-6, rtol=1e-6)


def test_maxpool_bwd_tie_rule():
    """Constant input: every window's first element (row-major) takes the gradient."""
    x = torch.ones(1, 4, 4, 1)
    dy = torch.ones(1, 2, 2, 1)
    dx = om.maxpool3x3s2_bwd(x, dy)[0, :, :, 0]
    # windows (pad 1, stride 2): output (0,0) covers rows/cols -1..1 -> first valid (0,0);
    # (0,1) covers cols 1..3 -> (0,1); (1,0) -> (1,0); (1,1) -> (1,1)
    ref = torch.zeros(4, 4)
    ref[0, 0] = ref[0, 1] = ref[1, 0] = ref[1, 1] = 1.0
    torch.testing.assert_close(dx, ref)


# --------------------------------------------------------------------------- ResNet training
def test_resnet_train_step_vs_torchvision():
    """ResNet-50-structured net with one bottleneck per stage (64x64 input, batch 4, 10
    classes): loss, every gradient, BN running stats and SGD(momentum) against torchvision's
    model + fp64 autograd."""
    tv = pytest.importorskip("torchvision")
    layers = [(64, 1, 1), (128, 1, 2), (256, 1, 2), (512, 1, 2)]
    spec = om.resnet_train_spec(layers, num_classes=10)
    P = si.make_params(spec)
    m = tv.models.resnet.ResNet(tv.models.resnet.Bottleneck, [1, 1, 1, 1], num_classes=10).double().train()
    _to_tv(P, m, _rn_rename)
    x = si.normal((4, 64, 64, 3), 2)
    lab = si.labels(4, 10, 2)
    loss, newP, newV, g = om.resnet_train_step(P, {}, x, lab, first=True, layers=layers)
    out = m(x.double().permute(0, 3, 1, 2))
    L = torch.nn.functional.cross_entropy(out, lab.long())
    L.backward()
    assert abs(float(loss) - float(L)) < 1e-5 * float(L)
    named, bufs = dict(m.named_parameters()), dict(m.named_buffers())
    assert set(_rn_rename(k) for k in g) == set(named)
    for k in g:
        ref = named[_rn_rename(k)].grad
        if ref.dim() == 4:
            ref = ref.permute(0, 2, 3, 1)
        err = float((g[k].double() - ref).norm() / max(float(ref.norm()), 1e-3))
        assert err < 1e-3, (k, err)
    for k in P:
        if k.endswith((".rmean", ".rvar")):
            torch.testing.assert_close(newP[k].double(), bufs[_rn_rename(k)], rtol=1e-5, atol=1e-6)
    k = "fc.w"
    torch.testing.assert_close(newP[k].double(), P[k].double() - 0.01 * named[_rn_rename(k)].grad, rtol=1e-5, atol=1e-7)


# ------------------------------------------------------------------------------------ col2im
@pytest.mark.parametrize("stride,pad,k", [(2, 1, 3), (2, 0, 1), (1, 1, 3), (2, 3, 7)])
def test_col2im_is_conv_data_gradient(stride, pad, k):
    """col2im(dy W) equals the convolution data gradient (adjoint identity), and an explicit loop."""
    n, h, w, c, kout = 2, 9, 8, 4, 5
    p, q = (h + 2 * pad - k) // stride + 1, (w + 2 * pad - k) // stride + 1
    dy = _rand(n, p, q, kout, seed=71)
    wt = _rand(kout, k, k, c, seed=72)
    col = (dy.double().reshape(-1, kout) @ wt.double().reshape(kout, -1))
    dx = om.col2im(col, (n, h, w, c), k, k, stride, pad)
    ref = om.conv2d_bwd_data(dy, wt, (n, h, w, c), stride, pad)
    torch.testing.assert_close(dx.double(), ref.double(), atol=1e-5, rtol=1e-5)
    colv = col.view(n, p, q, k, k, c)
    loop = torch.zeros(n, h, w, c, dtype=D)
    for b in range(n):
        for i in range(p):
            for j in range(q):
                for r in range(k):
                    for s in range(k):
                        hh, ww = i * stride - pad + r, j * stride - pad + s
                        if 0 <= hh < h and 0 <= ww < w:
                            loop[b, hh, ww] += colv[b, i, j, r, s]
    torch.testing.assert_close(dx.double(), loop, atol=1e-5, rtol=1e-5)


# ------------------------------------------------------------- Transformer encoder training
def test_layernorm_bwd_fd():
    x = _rand(5, 12, seed=81, dtype=D) * 2 + 1
    gm, bt = _rand(12, seed=82, dtype=D), _rand(12, seed=83, dtype=D)
    dy = _rand(5, 12, seed=84, dtype=D)
    y, m, r = om.layernorm_fwd(x, gm, bt)
    dx, dg, db = om.layernorm_bwd(x, dy, gm, m.double(), r.double())
    xr = x.clone().requires_grad_(True)
    gr, br = gm.clone().requires_grad_(True), bt.clone().requires_grad_(True)
    torch.nn.functional.layer_norm(xr, (12,), gr, br, 1e-5).backward(dy)
    torch.testing.assert_close(dx.double(), xr.grad, atol=2e-6, rtol=2e-5)
    torch.testing.assert_close(dg.double(), gr.grad, atol=2e-6, rtol=2e-5)
    torch.testing.assert_close(db.double(), br.grad, atol=2e-6, rtol=2e-5)


def test_mha_bwd_vs_autograd():
    B, S, heads, d = 2, 5, 2, 3
    q, k, v, do = (_rand(B, S, heads * d, seed=s, dtype=D) for s in (85, 86, 87, 88))
    dq, dk, dv = om.mha_bwd(q, k, v, do, heads)
    qr, kr, vr = (t.clone().requires_grad_(True) for t in (q, k, v))
    om_out = []

    def f(q_, k_, v_):
        Q, K, V = (t.view(B, S, heads, d).permute(0, 2, 1, 3) for t in (q_, k_, v_))
        o = torch.softmax(Q @ K.transpose(-1, -2) / math.sqrt(d), -1) @ V
        return o.permute(0, 2, 1, 3).reshape(B, S, heads * d)
    f(qr, kr, vr).backward(do)
    for a, b_ in ((dq, qr.grad), (dk, kr.grad), (dv, vr.grad)):
        torch.testing.assert_close(a.double(), b_, atol=1e-6, rtol=1e-5)


def test_encoder_train_step_vs_torch():
    """2-layer post-LN encoder (d 32, 4 heads, FFN 64), batch 2, seq 6: loss, every gradient and
    the SGD update against torch.nn.TransformerEncoderLayer in fp64 with autograd."""
    L_, dm, heads, ffn = 2, 32, 4, 64
    P = si.make_params(om.encoder_spec(L_, dm, ffn))
    x, t = si.normal((2, 6, dm), si.BE_SEED, sub=1), si.normal((2, 6, dm), si.BE_SEED, sub=2)
    loss, newP, _, g = om.encoder_train_step(P, {}, x, t, first=True, layers=L_, heads=heads)
    mods = [torch.nn.TransformerEncoderLayer(dm, heads, ffn, dropout=0.0, activation="relu", batch_first=True,
                                             norm_first=False).double() for _ in range(L_)]
    names = {"in.w": "self_attn.in_proj_weight", "in.b": "self_attn.in_proj_bias", "out.w": "self_attn.out_proj.weight",
             "out.b": "self_attn.out_proj.bias", "ln1.gamma": "norm1.weight", "ln1.beta": "norm1.bias",
             "ff1.w": "linear1.weight", "ff1.b": "linear1.bias", "ff2.w": "linear2.weight", "ff2.b": "linear2.bias",
             "ln2.gamma": "norm2.weight", "ln2.beta": "norm2.bias"}
    for i, m in enumerate(mods):
        sd = m.state_dict()
        for k2, tk in names.items():
            sd[tk] = P[f"enc{i}.{k2}"].double()
        m.load_state_dict(sd)
    h = x.double()
    for m in mods:
        h = m(h)
    L = ((h - t.double()) ** 2).mean()
    L.backward()
    assert abs(float(loss) - float(L)) < 1e-5 * float(L)
    for i, m in enumerate(mods):
        named = dict(m.named_parameters())
        for k2, tk in names.items():
            ref = named[tk].grad
            err = float((g[f"enc{i}.{k2}"].double() - ref).norm() / max(float(ref.norm()), 1e-12))
            assert err < 1e-4, (i, k2, err)
    k2 = "enc0.ff1.w"
    torch.testing.assert_close(newP[k2].double(), P[k2].double() - 0.01 * dict(mods[0].named_parameters())["linear1.weight"].grad,
                               rtol=1e-5, atol=1e-7)


def test_encoder_infer_vs_torch():
    """Inf-inf BE client ("Transformer" inference, R32): the encoder forward vs
    torch.nn.TransformerEncoderLayer stack in eval mode, fp64."""
    L_, dm, heads, ffn = 2, 32, 4, 64
    P = si.make_params(om.encoder_spec(L_, dm, ffn))
    x = si.normal((2, 6, dm), si.BE_SEED, sub=3)
    y = om.encoder_infer(P, x, layers=L_, heads=heads)
    mods = [torch.nn.TransformerEncoderLayer(dm, heads, ffn, dropout=0.0, activation="relu", batch_first=True,
                                             norm_first=False).double().eval() for _ in range(L_)]
    names = {"in.w": "self_attn.in_proj_weight", "in.b": "self_attn.in_proj_bias", "out.w": "self_attn.out_proj.weight",
             "out.b": "self_attn.out_proj.bias", "ln1.gamma": "norm1.weight", "ln1.beta": "norm1.bias",
             "ff1.w": "linear1.weight", "ff1.b": "linear1.bias", "ff2.w": "linear2.weight", "ff2.b": "linear2.bias",
             "ln2.gamma": "norm2.weight", "ln2.beta": "norm2.bias"}
    for i, m in enumerate(mods):
        sd = m.state_dict()
        for k2, tk in names.items():
            sd[tk] = P[f"enc{i}.{k2}"].double()
        m.load_state_dict(sd)
    h = x.double()
    with torch.no_grad():
        for m in mods:
            h = m(h)
    assert float((y.double() - h.reshape(-1, dm)).norm() / h.norm()) < 1e-5
