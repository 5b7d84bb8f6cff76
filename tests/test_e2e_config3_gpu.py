"""End-to-end at BASELINE config 3's full sizes: HP BERT-base inference (batch 8, seq 128, bf16)
collocated with BE ResNet-50 training (batch 64, 224x224, fp32) under liborion on the GPU.
  * HP last hidden states of 4 requests vs the oracle (rel L2 2e-2, north_star's bf16 bar);
  * one BE training iteration (loss, every gradient, running stats, SGD-updated parameters) vs the
    fp64 oracle with the ReLU decisions taken on the GPU's own values;
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


def test_be_rn50_one_iteration_vs_oracle(cfg3):
    be, Prn = cfg3["be"], cfg3["Prn"]
    be.graph.params.reset()
    C.run_session(be=be, be_iters=1)
    G = be.graph.params
    masks = {k: v.cpu() for k, v in be.graph.relu_in.items()}
    loss, newP, _, g_ref = om.resnet_train_step(Prn, {}, cfg3["xs"][0], cfg3["labels"][0], first=True, masks=masks)
    assert rel(be.graph.loss, loss.reshape(1)) < 1e-5
    # BN betas: floored at the same BN's dgamma norm (the stem BN's beta gradient nearly cancels: a
    # per-channel shift of its output changes the loss only through the ReLU mask, because the
    # max-pool output feeds conv -> train-BN on both block-1 paths). The stem's gradients (conv weight:
    # 802816 products per weight; BN gamma / beta: 802816-row sums at the end of the longest backward
    # chain) are held to 1e-3 (measured 3.7e-4). DESIGN.md §8.
    worst = {}
    for n, r in g_ref.items():
        floor = float(g_ref[n.replace(".beta", ".gamma")].norm()) if n.endswith(".beta") else 1e-30
        worst[n] = rel(G.g[n], r, floor)
    print("worst decision-aligned gradient errors:", sorted(worst.items(), key=lambda x: -x[1])[:6])
    stem = ("conv1.w", "bn1.gamma", "bn1.beta")
    bad = {k: v for k, v in worst.items() if v > (1e-3 if k in stem else 3e-4)}
    assert not bad, sorted(bad.items(), key=lambda x: -x[1])[:10]
    for name in newP:
        floor = 1e-2 if name.endswith(".rmean") else 1e-30
        if name.endswith(".beta"):   # starts at 0: the update is -lr * grad, floored like the gradient above
            floor = 0.01 * float(g_ref[name.replace(".beta", ".gamma")].norm())
        tol = 1e-3 if name in stem else (3e-4 if name.endswith(".beta") else 1e-5)
        assert rel(G.p[name], newP[name], floor) < tol, name
    assert torch.equal(G.vflat, G.gflat)


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
