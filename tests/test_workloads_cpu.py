"""Op-list builders (workloads.py) on the CPU: structure only (no kernels run). Parameter specs
must equal the oracle's independently written specs; every kernel op must carry at least the
args its table entry needs, with non-null device pointers where the kernel dereferences them."""
import pytest
import torch

from oracle import model as om
from synth import inputs as si
from paper_conf_eurosys_stratimk24_b200 import workloads as W, _lib as L


def test_specs_match_oracle():
    assert W.mlp_spec() == om.mlp_spec()
    assert W.resnet_spec() == om.resnet_spec()
    assert W.mnv2_spec() == om.mnv2_spec()
    assert W.mnv2_blocks() == om.mnv2_blocks()
    assert W.bert_spec(layers=2) == om.bert_spec(layers=2)
    assert W.resnet_train_spec() == om.resnet_train_spec()
    assert W.resnet_train_spec(W.RESNET101_LAYERS) == om.resnet_train_spec(om.RESNET101_LAYERS)
    assert W.encoder_spec(2) == om.encoder_spec(2)
    assert W.mnv2_spec(eval_stats=True) == om.mnv2_spec(eval_stats=True)
    assert W.resnet_spec(W.RESNET101_LAYERS) == om.resnet_spec(om.RESNET101_LAYERS)
    assert W.bert_spec(layers=2, hidden=1024, heads=16, ffn=4096) == om.bert_spec(layers=2, hidden=1024, heads=16, ffn=4096)


def test_infinf_client_graphs():
    """Inf-inf BE inference clients: H2D input first, D2H output last, every kernel op well formed."""
    g = W.mnv2_infer_graph(si.make_params(W.mnv2_spec(10, eval_stats=True)), batch=1, hw=32, num_classes=10, device="cpu")
    _check(g)
    kern = [o for o in g.ops if isinstance(o[0], str)]
    assert g.ops[0][2] == "h2d_input" and g.ops[-1][2] == "d2h_logits"
    assert sum(1 for o in kern if o[0] == "bn_eval") == 52 and sum(1 for o in kern if o[0] == "dw_fwd") == 17
    assert sum(1 for o in kern if o[0] == "add") == 10
    e = W.encoder_infer_graph(si.make_params(W.encoder_spec(2)), batch=1, seq=32, layers=2, device="cpu")
    _check(e)
    assert [o[0] for o in e.ops if isinstance(o[0], str)].count("attention_f32") == 2
    assert e.ops[0][2] == "h2d_input" and e.ops[-1][2] == "d2h_output"


NARGS = {"gemm": 13, "colsum": 4, "relu": 3, "relu_bwd": 4, "relu6": 3, "relu6_bwd": 4, "add": 4, "mse": 6, "sgd": 6,
         "conv_fwd": 16, "conv_dgrad": 16, "conv_wgrad": 16, "dw_fwd": 14, "dw_dgrad": 14, "dw_wgrad": 16,
         "bn_eval": 9, "bn_stats": 11, "bn_apply": 8, "bn_bwd_reduce": 10, "bn_bwd_dx": 10, "maxpool": 8,
         "avgpool": 5, "avgpool_bwd": 5, "ce": 7, "gemm_bf16": 7, "attention": 9, "layernorm": 7, "gelu": 3, "add_bf16": 4,
         "embed": 9, "maxpool_bwd": 9, "col2im": 12, "layernorm_f32": 9, "layernorm_f32_bwd": 12, "attention_f32": 10,
         "attention_f32_bwd_dq": 12, "attention_f32_bwd_dkv": 13}


def _check(g):
    for fn, args, lab in g.ops:
        if isinstance(fn, str):
            assert fn in L.FN, fn
            assert len(args) >= NARGS[fn], (lab, fn, len(args))
            assert all(isinstance(a, int) for a in args), lab
            assert args[0] != 0, lab


def test_mlp_graphs():
    P = si.make_params(W.mlp_spec(64))
    hp = W.mlp_infer_graph(P, batch=1, width=64, device="cpu")
    assert [o[2] for o in hp.ops] == ["h2d_input", "fc0", "relu0", "fc1", "relu1", "fc2", "d2h_output"]
    _check(hp)
    xs = [si.normal((4, 64), 2, sub=i) for i in range(2)]
    be = W.mlp_train_graph(P, xs, xs, width=64, device="cpu")
    assert len(be.variants) == 2 and len(be.variants[0]) == len(be.variants[1]) == 17
    for v in be.variants:
        be.ops = v
        _check(be)


def test_resnet_graph_structure():
    P = si.make_params(W.resnet_spec())
    g = W.resnet_infer_graph(P, batch=1, hw=32, device="cpu")
    _check(g)
    labs = [o[2] for o in g.ops]
    kern = [o for o in g.ops if isinstance(o[0], str)]
    # 53 convs (+ fc), 53 BN, 49 ReLU, 16 add, maxpool, avgpool -> 174 ops + 2 memops
    assert sum(1 for o in kern if o[2].endswith(".relu") or o[2] == "bn1.relu") == 49
    assert sum(1 for o in kern if o[0] == "bn_eval") == 53
    assert sum(1 for o in kern if o[0] == "add") == 16
    assert len(kern) == 174, len(kern)
    assert labs[0] == "h2d_input" and labs[-1] == "d2h_logits"


def test_mnv2_graph_structure():
    P = si.make_params(W.mnv2_spec(num_classes=10))
    xs = [si.normal((2, 32, 32, 3), 2, sub=i) for i in range(2)]
    labels = [si.labels(2, 10, 2, sub=i) for i in range(2)]
    g = W.mnv2_train_graph(P, xs, labels, num_classes=10, device="cpu")
    assert len(g.variants) == 2
    for v in g.variants:
        g.ops = v
        _check(g)
    fns = [o[0] for o in g.variants[0]]
    assert fns.count("bn_stats") == 52 and fns.count("bn_bwd_dx") == 52
    assert fns.count("sgd") == 1 and fns.count("ce") == 1
    assert fns.count("dw_fwd") == 17 and fns.count("dw_wgrad") == 17 and fns.count("dw_dgrad") == 17
    assert 350 <= len(fns) <= 520, len(fns)


def test_variants_share_one_live_workspace():
    """Every variant's ops must point at the one workspace the graph keeps alive (a freed workspace
    would be reused by the allocator: a dangling-pointer race)."""
    P = si.make_params(W.mnv2_spec(num_classes=10))
    xs = [si.normal((2, 32, 32, 3), 2, sub=i) for i in range(3)]
    labels = [si.labels(2, 10, 2, sub=i) for i in range(3)]
    g = W.mnv2_train_graph(P, xs, labels, num_classes=10, device="cpu")
    ws = g._ws.data_ptr()
    for v in g.variants:
        for fn, args, lab in v:
            if fn in ("bn_stats", "dw_wgrad", "ce", "conv_wgrad"):
                at = {"bn_stats": 9, "dw_wgrad": 14, "ce": 6, "conv_wgrad": 14}[fn]
                assert args[at] == ws, lab
    Pm = si.make_params(W.mlp_spec(64))
    xm = [si.normal((4, 64), 2, sub=i) for i in range(3)]
    gm = W.mlp_train_graph(Pm, xm, xm, width=64, device="cpu")
    for v in gm.variants:
        for fn, args, lab in v:
            if fn == "mse":
                assert args[5] == gm._ws.data_ptr()


def test_graph_buffers_never_replaced():
    """Op lists hold raw device pointers: a second request for a named buffer (e.g. a per-op scratch
    built once per op-list variant) must return the same tensor, never free the first one."""
    from paper_conf_eurosys_stratimk24_b200 import workloads as W
    g = W.Graph("t", device="cpu")
    a = g.buf("col.x", (4, 4))
    b = g.buf("col.x", (4, 4))
    assert a.data_ptr() == b.data_ptr()
    import pytest
    with pytest.raises(AssertionError):
        g.buf("col.x", (2, 4))


def test_config3_config4_graphs():
    """BERT (bf16), ResNet-50 / -101 training and the encoder: every op carries its args, the HP
    graphs start with an H2D and end with a D2H memop, and the analytic work of every op is defined
    (the profiler's roofline / classifier needs it)."""
    from paper_conf_eurosys_stratimk24_b200 import profiler as PR
    gb = W.bert_infer_graph(si.make_params(W.bert_spec(layers=2)), batch=2, seq=32, layers=2, device="cpu")
    gr = W.resnet_train_graph(si.make_params(W.resnet_train_spec()), [si.normal((1, 64, 64, 3), 2)], [si.labels(1, 1000, 2)], device="cpu")
    ge = W.encoder_train_graph(si.make_params(W.encoder_spec(2)), [si.normal((2, 32, 512), 2)], [si.normal((2, 32, 512), 3)],
                               layers=2, device="cpu")
    x = si.normal((1, 64, 64, 3), 1)
    gh = W.as_hp_training(W.resnet_train_graph(si.make_params(W.resnet_train_spec(W.RESNET101_LAYERS)), [x], [si.labels(1, 1000, 1)],
                                               layers=W.RESNET101_LAYERS, device="cpu"), x)
    for g in (gb, gr, ge, gh):
        _check(g)
        for i, fn, args, lab in g.kernel_ops():
            flops, nbytes = PR.op_work(fn, args)
            assert nbytes > 0, (lab, fn)
    for g in (gb, gh):
        assert g.ops[0][0] == L.OP_MEMCPY_H2D and g.ops[-1][0] == L.OP_MEMCPY_D2H
