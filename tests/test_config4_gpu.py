"""BASELINE config 4 (train-train): HP ResNet-101 training (throughput mode) collocated with BE
post-LN Transformer-encoder training (fp32) under liborion.
  * teacher-forced per-op parity of the encoder's op list at full width (d 512, 8 heads, FFN 2048,
    batch 8, seq 192; 2 layers) vs the fp64 oracle ops (2e-5);
  * two encoder iterations end to end vs the oracle, and two full-size ResNet-101 b32 HP training
    iterations vs the oracle, ReLU decisions audited (tests/parity.py);
  * a collocated session (HP ResNet-101 at a reduced batch): decision log == oracle replay byte for
    byte, HP and BE parameters bitwise identical to solo runs of the same iteration counts."""
import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import policy_ffi as po
from synth import inputs as si
import logfmt as lf

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_eurosys_stratimk24_b200 as orion
    from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C, profiler as PR
    import opcheck


def rel(a, b, floor=1e-30):
    a, b = torch.as_tensor(a).double().cpu(), torch.as_tensor(b).double().cpu()
    return float((a - b).norm() / max(float(b.norm()), floor))


def _enc(layers=2, b=8, s=192):
    P = si.make_params(W.encoder_spec(layers))
    xs = [si.normal((b, s, 512), si.BE_SEED, sub=i) for i in range(2)]
    ts = [si.normal((b, s, 512), si.BE_SEED, sub=50 + i) for i in range(2)]
    return P, xs, ts, W.encoder_train_graph(P, xs, ts, layers=layers)


def test_encoder_spec_matches_oracle():
    assert W.encoder_spec(3) == om.encoder_spec(3)


def test_encoder_ops_teacher_forced():
    P, xs, ts, g = _enc()
    Pm = g.params
    tensors = [Pm.flat] + list(g.bufs.values()) + list(Pm.p.values()) + list(Pm.g.values()) + [g._ws]
    R = opcheck.Resolver(tensors)
    R_in = opcheck.Resolver(tensors, read_alias={Pm.flat.data_ptr(): Pm.flat.clone()})
    s = torch.cuda.current_stream().cuda_stream
    errs = []
    for i, (fn, args, lab) in enumerate(g.ops):   # gradient buffers are shared across layers: check each op right away
        orion.kernel_launch(fn, args, s)
        torch.cuda.synchronize()
        if fn == "sgd":
            continue
        e = opcheck.check_op(fn, args, R, None, R_in)
        assert e is not None, fn
        errs.append((e, i, lab, fn))
    for e in sorted(errs, reverse=True)[:6]:
        print("encoder", e)
    bad = [e for e in errs if e[0] > 2e-5]
    assert not bad, sorted(bad, reverse=True)[:10]


def test_encoder_iterations_vs_oracle():
    """K = 2 encoder iterations (2 layers at full width) vs the fp64 oracle, the GPU's FFN ReLU
    decisions audited against the oracle's own pre-activations (tests/parity.py)."""
    import copy
    import parity as PT
    P, xs, ts, g = _enc()
    be = C.BEClient(g)
    g.params.reset()

    def run_one(it):
        one = copy.copy(be)
        one.variants = [be.variants[it]]
        C.run_session(be=one, be_iters=1)

    def step(Pp, V, x, t, first, masks, trace):
        return om.encoder_train_step(Pp, V, x, t, first=first, layers=2, masks=masks, trace=trace)
    rep = PT.check_train_iterations(run_one, g, step, xs, ts, P, 2, "relu_in", (0.0,), trace_order="backward")
    print("encoder iterations vs oracle:", rep)


def test_rn101_hp_training_full_size_vs_oracle():
    """Config 4's HP at its full size: one ResNet-101 training iteration at batch 32, 224x224 (the
    HP op list the train-train bench runs) vs the fp64 oracle with audited ReLU decisions
    (tests/parity.py). One iteration: the fp32 forward of a 101-layer train-mode network drifts
    ~8 % per block from the fp64 one (5e-4 at layer4); after one SGD step the second forward
    amplifies that parameter difference to a few percent, so a second iteration measures the
    network's sensitivity, not the kernels."""
    import copy
    import parity as PT
    torch.cuda.set_device(0)
    Pr = si.make_params(W.resnet_train_spec(W.RESNET101_LAYERS))
    xs = [si.normal((32, 224, 224, 3), si.HP_SEED, sub=i) for i in range(2)]
    labs = [si.labels(32, 1000, si.HP_SEED, sub=i) for i in range(2)]
    hpg = W.resnet_train_graph(Pr, xs, labs, layers=W.RESNET101_LAYERS)
    be = C.BEClient(hpg)
    hpg.params.reset()

    def run_one(it):
        one = copy.copy(be)
        one.variants = [be.variants[it]]
        C.run_session(be=one, be_iters=1)

    def step(Pp, V, x, lab, first, masks, trace):
        return om.resnet_train_step(Pp, V, x, lab, first=first, layers=W.RESNET101_LAYERS, masks=masks, trace=trace)
    rep = PT.check_train_iterations(run_one, hpg, step, xs, labs, Pr, 1, "relu_in", (0.0,), trace_order="backward")
    print("ResNet-101 b32 training iteration vs oracle:", rep)


def test_rn101_hp_encoder_be_collocated():
    Pr = si.make_params(W.resnet_train_spec(W.RESNET101_LAYERS))
    x = si.normal((4, 112, 112, 3), si.HP_SEED)
    hpg = W.resnet_train_graph(Pr, [x], [si.labels(4, 1000, si.HP_SEED)], layers=W.RESNET101_LAYERS)
    W.as_hp_training(hpg, x)
    P, xs, ts, beg = _enc(layers=2, b=4, s=64)
    ph, _ = PR.build_profiles(hpg, 0, reps=2)
    pb, _ = PR.build_profiles(beg, 10000, reps=2)
    hpg.params.reset()
    beg.params.reset()
    hp = C.HPClient(hpg, [x], 6, ph, 0)
    be = C.BEClient(beg, pb, 10000)
    res = C.run_session(hp=hp, be=be, arrivals_ns=np.zeros(6, dtype=np.int64), log_capacity=1 << 22, hp_latency_ns=5_000_000)
    _, prefix, _, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    K = len(res["be_t_end"])
    hp_col, be_col = hpg.params.flat.cpu().clone(), beg.params.flat.cpu().clone()
    hpg.params.reset()
    C.run_session(hp=hp, arrivals_ns=np.zeros(6, dtype=np.int64))
    assert torch.equal(hpg.params.flat.cpu(), hp_col)
    beg.params.reset()
    if K:
        C.run_session(be=be, be_iters=K)
        assert torch.equal(beg.params.flat.cpu(), be_col)
