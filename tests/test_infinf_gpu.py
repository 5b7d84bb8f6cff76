"""SURVEY §8(f) row 3 / PAPER.md §6.3 (Fig. 13): one HP and four BE *inference*
clients on one GPU, every one open-loop Poisson (Table 3 "Inf-Inf Poisson" rates, Table 1 batch
sizes; reading R34): HP ResNet-50 b4 with BE MobileNetV2 b4, ResNet-101 b4, BERT-large b2 (bf16)
and the Transformer encoder b4, at their full sizes, under liborion.
  * every client's outputs vs the fp64 oracle (fp32 clients rel L2 1e-4, elementwise 10x; BERT
    2e-2, north_star's bf16 bar);
  * decision log == oracle replay, byte for byte (four BE clients rotate, R11);
  * every client's outputs bitwise identical between the collocated run and its solo run."""
import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import policy_ffi as po
from synth import inputs as si
import logfmt as lf
import parity as PT

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import bench
    from paper_conf_eurosys_stratimk24_b200 import collocate as C, profiler as PR, workloads as W

N_REQ = 4


def _oracle(name, P, x):
    if name in ("resnet50", "resnet101"):
        return om.resnet_infer(P, x, om.RESNET50_LAYERS if name == "resnet50" else om.RESNET101_LAYERS)
    if name == "mobilenet_v2":
        return om.mnv2_infer(P, x)
    if name == "bert_large":
        return om.bert_infer(om.to_model_dtype(P), x.view(torch.int32).view(2, 128), layers=24, heads=16)
    return om.encoder_infer(P, x)


@pytest.fixture(scope="module")
def infinf():
    torch.cuda.set_device(0)
    clients = []
    for j, (name, rps) in enumerate(bench.INFINF):
        g, xs, P, view = bench.build_infinf_client(name, n_inputs=N_REQ)
        prof, _ = PR.build_profiles(g, 10000 * j, reps=2)
        clients.append(dict(name=name, rps=rps, P=P, xs=xs, view=view, c=C.HPClient(g, xs, N_REQ, prof, 10000 * j)))
    return clients


def test_infinf_outputs_log_and_solo(infinf):
    hp, bes = infinf[0], infinf[1:]
    # arrivals at 4x Table 3's rates keep the run short while the clients still overlap
    arr = [si.poisson_arrivals_ns(4 * cl["rps"], N_REQ, seed=si.ARRIVAL_SEED + j) for j, cl in enumerate(infinf)]
    for cl in infinf:
        cl["c"].out.zero_()
    res = C.run_inference_session(hp=hp["c"], hp_arrivals=arr[0], bes=[b["c"] for b in bes], be_arrivals=arr[1:],
                                  log_capacity=1 << 22, hp_latency_ns=3_000_000)
    _, prefix, _, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    kinds = {d[1] for d in lf.decode_decisions(decs)}
    assert 4 in kinds or 3 in kinds      # BE requests admitted (beside the HP or while it is idle)
    col = [cl["c"].out.clone() for cl in infinf]
    for cl, out in zip(infinf, col):
        for r in range(N_REQ):
            got, ref = cl["view"](out[r]), _oracle(cl["name"], cl["P"], cl["xs"][r])
            if cl["name"] == "bert_large":
                e = PT.rel(got, ref)
                assert e < 2e-2, (cl["name"], r, e)
            else:
                PT.assert_close(f"{cl['name']} request {r}", got, ref, 1e-4)
    # solo runs: each client alone reproduces its collocated outputs bit for bit
    for j, cl in enumerate(infinf):
        cl["c"].out.zero_()
        if j == 0:
            C.run_inference_session(hp=cl["c"], hp_arrivals=arr[0])
        else:
            C.run_inference_session(bes=[cl["c"]], be_arrivals=[arr[j]])
        assert torch.equal(cl["c"].out, col[j]), cl["name"]
