"""Teacher-forced per-op parity of the full client op lists at BASELINE config 2's sizes, launched
through the C ABI in op-list order: every op's output vs the fp64 oracle op applied to the GPU's
own inputs (tests/opcheck.py). Catches wiring mistakes (wrong buffer, stride, flag) that a single-op
unit test cannot, at full size, op by op."""
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


def _run_and_check(g, extra_tensors, every=1, report=None):
    s = torch.cuda.current_stream().cuda_stream
    P = g.params
    tensors = [P.flat] + list(g.bufs.values()) + list(P.p.values()) + list(P.g.values()) + extra_tensors + [g._ws]
    R = opcheck.Resolver(tensors)
    R_in = opcheck.Resolver(tensors, read_alias={P.flat.data_ptr(): P.flat.clone()})
    snaps = {}
    for i, (fn, args, lab) in enumerate(g.ops):
        if not isinstance(fn, str):
            continue
        if fn == "bn_stats":
            snaps[i] = {args[3]: R.get(args[3], args[6]).cpu().clone(), args[4]: R.get(args[4], args[6]).cpu().clone()}
        orion.kernel_launch(fn, args, s)
    torch.cuda.synchronize()
    errs = []
    for i, (fn, args, lab) in enumerate(g.ops):
        if not isinstance(fn, str) or fn == "sgd" or (i % every and fn not in ("ce", "bn_stats")):
            continue
        e = opcheck.check_op(fn, args, R, snaps.get(i), R_in)
        if e is not None:
            errs.append((e, i, lab, fn))
    if report:
        for e in sorted(errs, reverse=True)[:15]:
            print(report, e)
    return errs


def test_mnv2_train_ops_teacher_forced():
    hw, b = (224, 96) if FULL else (112, 16)
    P = si.make_params(W.mnv2_spec())
    xs = [si.normal((b, hw, hw, 3), si.BE_SEED, sub=0)]
    labels = [si.labels(b, 1000, si.BE_SEED, sub=0)]
    g = W.mnv2_train_graph(P, xs, labels)
    errs = _run_and_check(g, [], every=1, report="mnv2")
    bad = [e for e in errs if e[0] > 2e-5]
    assert not bad, sorted(bad, reverse=True)[:10]


def test_resnet50_infer_ops_teacher_forced():
    P = si.make_params(W.resnet_spec())
    g = W.resnet_infer_graph(P, batch=4)
    g.x.copy_(si.normal((4, 224, 224, 3), si.HP_SEED).cuda())
    errs = _run_and_check(g, [], report="rn50")
    bad = [e for e in errs if e[0] > 2e-5]
    assert not bad, sorted(bad, reverse=True)[:10]


def test_mnv2_train_ops_full_size():
    """BASELINE config 2's BE client at its full size (MobileNetV2 b96, 224x224): the whole op list
    runs through the C ABI in order and every op is checked teacher-forced against the fp64 oracle op
    on the GPU's own inputs -- the launch configurations the bench times, at sizes the reduced-size
    test above does not reach."""
    P = si.make_params(W.mnv2_spec())
    xs = [si.normal((96, 224, 224, 3), si.BE_SEED, sub=0)]
    labels = [si.labels(96, 1000, si.BE_SEED, sub=0)]
    g = W.mnv2_train_graph(P, xs, labels)
    errs = _run_and_check(g, [], every=1, report="mnv2-full")
    bad = [e for e in errs if e[0] > 2e-5]
    assert len(errs) >= 400, len(errs)
    assert not bad, sorted(bad, reverse=True)[:10]
