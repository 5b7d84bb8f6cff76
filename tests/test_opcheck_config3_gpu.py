"""Teacher-forced per-op parity of config 3's client op lists (HP BERT-base bf16 inference at its
full size, BE ResNet-50 training at a reduced batch), launched through the C ABI in op-list order:
every op's output vs the fp64 oracle op applied to the GPU's own inputs (tests/opcheck.py).
Tolerances: bf16 ops 5e-3 (one bf16 rounding on each side, attention's P rounding), fp32 ops 2e-5
(DESIGN.md §8)."""
import os

import pytest
import torch

from synth import inputs as si

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_eurosys_stratimk24_b200 as orion
    from paper_conf_eurosys_stratimk24_b200 import workloads as W
    import opcheck

FULL = os.environ.get("ORION_OPCHECK_FULL", "0") == "1"
BF16_OPS = ("gemm_bf16", "attention", "layernorm", "gelu", "add_bf16", "embed")


def _launch_all(g, snaps_for=()):
    s = torch.cuda.current_stream().cuda_stream
    snaps = {}
    for i, (fn, args, lab) in enumerate(g.ops):
        if not isinstance(fn, str):
            continue
        if fn == "bn_stats":
            snaps[i] = {args[3]: snaps_for.get(args[3], args[6]).cpu().clone(), args[4]: snaps_for.get(args[4], args[6]).cpu().clone()}
        orion.kernel_launch(fn, args, s)
    torch.cuda.synchronize()
    return snaps


def test_bert_infer_ops_teacher_forced():
    P = si.make_params(W.bert_spec())
    g = W.bert_infer_graph(P, batch=8, seq=128)
    g.x.copy_(si.token_ids((8, 128), 30522, si.HP_SEED).reshape(-1).cuda())
    tensors = list(g.bufs.values())
    R = opcheck.Resolver(tensors)
    _launch_all(g, R)
    errs = []
    for i, (fn, args, lab) in enumerate(g.ops):
        if isinstance(fn, str):
            errs.append((opcheck.check_op(fn, args, R), i, lab, fn))
    for e in sorted(errs, reverse=True)[:8]:
        print("bert", e)
    assert all(e[0] is not None for e in errs)
    bad = [e for e in errs if e[0] > 5e-3]
    assert not bad, sorted(bad, reverse=True)[:10]


def test_resnet50_train_ops_teacher_forced():
    hw, b = (224, 64) if FULL else (112, 4)
    P = si.make_params(W.resnet_train_spec())
    g = W.resnet_train_graph(P, [si.normal((b, hw, hw, 3), si.BE_SEED, sub=0)], [si.labels(b, 1000, si.BE_SEED, sub=0)])
    Pm = g.params
    tensors = [Pm.flat] + list(g.bufs.values()) + list(Pm.p.values()) + list(Pm.g.values()) + [g._ws]
    R = opcheck.Resolver(tensors)
    R_in = opcheck.Resolver(tensors, read_alias={Pm.flat.data_ptr(): Pm.flat.clone()})
    snaps = _launch_all(g, R)
    errs = []
    for i, (fn, args, lab) in enumerate(g.ops):
        if not isinstance(fn, str) or fn == "sgd":
            continue
        e = opcheck.check_op(fn, args, R, snaps.get(i), R_in)
        assert e is not None, fn
        errs.append((e, i, lab, fn))
    for e in sorted(errs, reverse=True)[:8]:
        print("rn50 train", e)
    bad = [e for e in errs if e[0] > 2e-5]
    assert not bad, sorted(bad, reverse=True)[:10]


def test_resnet50_train_ops_full_size_sampled():
    """Config 3's BE client at its full size (ResNet-50 training b64, 224x224): the whole op list runs
    through the C ABI in order; every 8th op plus every loss / BN-statistics op is checked
    teacher-forced against the fp64 oracle op (all ops at full size would take ~10 min of fp64 CPU)."""
    P = si.make_params(W.resnet_train_spec())
    g = W.resnet_train_graph(P, [si.normal((64, 224, 224, 3), si.BE_SEED, sub=0)], [si.labels(64, 1000, si.BE_SEED, sub=0)])
    Pm = g.params
    tensors = [Pm.flat] + list(g.bufs.values()) + list(Pm.p.values()) + list(Pm.g.values()) + [g._ws]
    R = opcheck.Resolver(tensors)
    R_in = opcheck.Resolver(tensors, read_alias={Pm.flat.data_ptr(): Pm.flat.clone()})
    snaps = _launch_all(g, R)
    errs = []
    for i, (fn, args, lab) in enumerate(g.ops):
        if not isinstance(fn, str) or fn == "sgd" or (i % 8 and fn not in ("ce", "bn_stats")):
            continue
        e = opcheck.check_op(fn, args, R, snaps.get(i), R_in)
        assert e is not None, fn
        errs.append((e, i, lab, fn))
    for e in sorted(errs, reverse=True)[:8]:
        print("rn50 train full", e)
    assert len(errs) >= 100, len(errs)
    bad = [e for e in errs if e[0] > 2e-5]
    assert not bad, sorted(bad, reverse=True)[:10]
