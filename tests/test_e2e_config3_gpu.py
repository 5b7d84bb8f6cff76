"""End-to-end at BASELINE config 3's full sizes: HP BERT-base inference (batch 8, seq 128, bf16)
collocated with BE ResNet-50 training (batch 64, 224x224, fp32) under liborion on the GPU.
  * HP last hidden states of 4 requests vs the oracle (rel L2 2e-2, north_star's bf16 bar);
  * K = 2 BE training iterations (loss, every gradient, momentum, running stats, parameters) vs the
    fp64 oracle, the GPU's ReLU decisions audited against the oracle's own;
  * decision log == oracle replay, byte for byte;
  * HP outputs and BE parameters bitwise identical between collocated and solo runs."""
import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import policy_ffi as po
from synth import inputs as si
import logfmt as lf

pytestmark = pytest.mark.gpu
BF = torch.bfloat16

if torch.cuda.is_available():
    from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C, profiler as PR


def rel(a, b, floor=1e-30):
    a, b = torch.as_tensor(a).double().cpu(), torch.as_tensor(b).double().cpu()
    return float((a - b).norm() / max(float(b.norm()), floor))


@pytest.fixture(scope="module")
def cfg3():
    torch.cuda.set_device(0)
    Pb = si.make_params(W.bert_spec())
    ids = [si.token_ids((8, 128), 30522, si.HP_SEED, sub=r) for r in range(4)]
    hpg = W.bert_infer_graph(Pb, batch=8, seq=128)
    Prn = si.make_params(W.resnet_train_spec())
    xs = [si.normal((64, 224, 224, 3), si.BE_SEED, sub=i) for i in range(2)]
    labels = [si.labels(64, 1000, si.BE_SEED, sub=i) for i in range(2)]
    beg = W.resnet_train_graph(Prn, xs, labels)
    ph, _ = PR.build_profiles(hpg, 0, reps=3)
    pb, _ = PR.build_profiles(beg, 10000, reps=3)
    beg.params.reset()
    hp = C.HPClient(hpg, [t.reshape(-1).view(torch.float32) for t in ids], 8, ph, 0)
    be = C.BEClient(beg, pb, 10000)
    lat = C.latency_stats(C.run_session(hp=hp, arrivals_ns=(np.arange(1, 11) * 20e6).astype(np.int64)))["p50_ns"]
    return dict(Pb=Pb, Prn=Prn, hp=hp, be=be, ids=ids, xs=xs, labels=labels, lat=int(lat))


def _hidden(hp, r):
    return hp.out[r].view(BF).view(8, 128, 768)


def test_hp_bert_vs_oracle(cfg3):
    hp = cfg3["hp"]
    hp.out.zero_()
    C.run_session(hp=hp, arrivals_ns=(np.arange(1, 5) * 10e6).astype(np.int64))
    Pbf = om.to_model_dtype(cfg3["Pb"])
    for r in range(4):
        ref = om.bert_infer(Pbf, cfg3["ids"][r])
        e = rel(_hidden(hp, r), ref)
        print("bert request", r, "rel L2", e)
        assert e < 2e-2, (r, e)


def test_be_rn50_iterations_vs_oracle(cfg3):
    """K = 2 BE ResNet-50 b64 training iterations vs the fp64 oracle, the GPU's ReLU decisions
    (BN outputs and residual sums) and max-pool maxima audited against the oracle's own forward
    (tests/parity.py, check_train_iterations)."""
    import copy
    import parity as PT
    be, Prn = cfg3["be"], cfg3["Prn"]
    be.graph.params.reset()

    def run_one(it):
        one = copy.copy(be)
        one.variants = [be.variants[it]]
        C.run_session(be=one, be_iters=1)

    def step(P, V, x, lab, first, masks, trace):
        return om.resnet_train_step(P, V, x, lab, first=first, masks=masks, trace=trace)
    rep = PT.check_train_iterations(run_one, be.graph, step, cfg3["xs"], cfg3["labels"], Prn, 2, "relu_in", (0.0,),
                                    trace_order="backward")
    print("ResNet-50 b64 BE iterations vs oracle:", rep)


def test_collocated_parity_and_log(cfg3):
    hp, be = cfg3["hp"], cfg3["be"]
    be.graph.params.reset()
    hp.out.zero_()
    arrivals = si.poisson_arrivals_ns(20.0, 8)
    res = C.run_session(hp=hp, be=be, arrivals_ns=arrivals, log_capacity=1 << 22, hp_latency_ns=cfg3["lat"])
    out_col = hp.out.clone()
    K = len(res["be_t_end"])
    p_col = be.graph.params.flat.cpu().clone()
    assert K >= 1
    _, prefix, _, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    hp.out.zero_()
    C.run_session(hp=hp, arrivals_ns=arrivals)
    assert torch.equal(hp.out, out_col)
    be.graph.params.reset()
    C.run_session(be=be, be_iters=K)
    assert torch.equal(be.graph.params.flat.cpu(), p_col)
