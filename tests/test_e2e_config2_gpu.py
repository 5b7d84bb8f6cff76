"""End-to-end at BASELINE config 2's full sizes: HP ResNet-50 inference b4 (224x224) collocated with
BE MobileNetV2 training b96 under liborion on the GPU, in the bench's launch configuration.
  * HP logits of 16 requests vs the fp64 oracle (rel L2 1e-4, north_star);
  * K = 3 BE training iterations (loss, every gradient, momentum, BN running stats, parameters) vs
    the fp64 oracle, with the GPU's ReLU6 decisions audited against the oracle's own forward and
    the error model of DESIGN.md §8 (tests/parity.py);
  * decision log == oracle replay, byte for byte;
  * HP logits and BE parameters bitwise identical between collocated and solo runs."""
import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import policy_ffi as po
from synth import inputs as si
import logfmt as lf

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C, profiler as PR


def rel(a, b, floor=1e-30):
    a, b = torch.as_tensor(a).double().cpu(), torch.as_tensor(b).double().cpu()
    return float((a - b).norm() / max(float(b.norm()), floor))


@pytest.fixture(scope="module")
def cfg2():
    torch.cuda.set_device(0)
    Prn = si.make_params(W.resnet_spec())
    hp_inputs = [si.normal((4, 224, 224, 3), si.HP_SEED, sub=r) for r in range(16)]
    hpg = W.resnet_infer_graph(Prn, batch=4)
    Pmn = si.make_params(W.mnv2_spec())
    xs = [si.normal((96, 224, 224, 3), si.BE_SEED, sub=i) for i in range(8)]
    labels = [si.labels(96, 1000, si.BE_SEED, sub=i) for i in range(8)]
    beg = W.mnv2_train_graph(Pmn, xs, labels)
    ph, _ = PR.build_profiles(hpg, 0, reps=3)
    pb, _ = PR.build_profiles(beg, 10000, reps=3)
    beg.params.reset()
    hp = C.HPClient(hpg, hp_inputs, 16, ph, 0)
    be = C.BEClient(beg, pb, 10000)
    lat = C.latency_stats(C.run_session(hp=hp, arrivals_ns=(np.arange(1, 11) * 30e6).astype(np.int64)))["p50_ns"]
    return dict(Prn=Prn, Pmn=Pmn, hp=hp, be=be, xs=xs, labels=labels, hp_inputs=hp_inputs, lat=int(lat))


K_ITERS = 3          # BE compared after K = 1 and K = 3 iterations


def test_be_iterations_vs_oracle(cfg2):
    """K = 3 BE training iterations (batches 0, 1, 2) on the GPU against the fp64 oracle, the GPU's
    ReLU6 decisions audited against the oracle's own forward (tests/parity.py,
    check_train_iterations)."""
    import copy
    import parity as PT
    be, Pmn = cfg2["be"], cfg2["Pmn"]
    be.graph.params.reset()

    def run_one(it):
        one = copy.copy(be)
        one.variants = [be.variants[it]]          # batch `it`
        C.run_session(be=one, be_iters=1)

    def step(P, V, x, lab, first, masks, trace):
        return om.mnv2_train_step(P, V, x, lab, first=first, masks=masks, trace=trace)
    rep = PT.check_train_iterations(run_one, be.graph, step, cfg2["xs"], cfg2["labels"], Pmn, K_ITERS, "bn_out",
                                    (0.0, 6.0), audit_skip=("project_bn",))
    print("MobileNetV2 b96 BE iterations vs oracle:", rep)


def test_collocated_parity_and_log(cfg2):
    hp, be = cfg2["hp"], cfg2["be"]
    be.graph.params.reset()
    hp.out.zero_()
    arrivals = si.poisson_arrivals_ns(40.0, 16)
    res = C.run_session(hp=hp, be=be, arrivals_ns=arrivals, log_capacity=1 << 22, hp_latency_ns=cfg2["lat"])
    out_col = hp.out.clone()
    K = len(res["be_t_end"])
    p_col = be.graph.params.flat.cpu().clone()
    assert K >= 1
    # decision log bit-exact vs oracle replay of the recorded tape
    _, prefix, _, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    # HP logits vs oracle
    for r in range(16):
        ref = om.resnet_infer(cfg2["Prn"], cfg2["hp_inputs"][r])
        assert rel(out_col[r].view(4, 1000), ref) < 1e-4, r
    # solo runs: bitwise equal
    hp.out.zero_()
    C.run_session(hp=hp, arrivals_ns=arrivals)
    assert torch.equal(hp.out, out_col)
    be.graph.params.reset()
    C.run_session(be=be, be_iters=K)
    assert torch.equal(be.graph.params.flat.cpu(), p_col)
