"""End-to-end, config 1 (toy): HP 3x512 MLP inference b1 (200 Poisson requests) collocated with BE
MLP training b32 under liborion on the GPU.
  * decision log == oracle replay of the run's own tape, byte for byte (north_star);
  * every HP output and the BE parameters after K iterations match the fp64 oracle (rel L2 1e-4);
  * outputs are bitwise identical between the collocated run and solo runs."""
import numpy as np
import pytest
import torch

from oracle import model as om
from oracle import policy_ffi as po
from synth import inputs as si
import logfmt as lf

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C, profiler as PR, _lib as L


def rel(a, b):
    a, b = torch.as_tensor(a).double(), torch.as_tensor(b).double()
    return float((a - b).norm() / max(float(b.norm()), 1e-30))


@pytest.fixture(scope="module")
def toy():
    spec = W.mlp_spec()
    assert spec == om.mlp_spec()
    P = si.make_params(spec)
    n_req = 200
    xs_hp = [si.normal((1, 512), si.HP_SEED, sub=r) for r in range(n_req)]
    xs_be = [si.normal((32, 512), si.BE_SEED, sub=i) for i in range(8)]
    ts_be = [si.normal((32, 512), si.BE_SEED, sub=100 + i) for i in range(8)]
    hpg = W.mlp_infer_graph(P, batch=1)
    beg = W.mlp_train_graph(P, xs_be, ts_be, lr=0.01)
    prof_hp, _ = PR.build_profiles(hpg, kid_base=0, reps=5)
    prof_be, _ = PR.build_profiles(beg, kid_base=1000, reps=5)
    beg.params.reset()
    hp = C.HPClient(hpg, xs_hp, n_req, prof_hp, 0)
    be = C.BEClient(beg, prof_be, 1000)
    arrivals = si.poisson_arrivals_ns(1000.0, n_req)
    return dict(P=P, hp=hp, be=be, arrivals=arrivals, xs_hp=xs_hp, xs_be=xs_be, ts_be=ts_be)


def test_toy_collocated_parity(toy):
    hp, be = toy["hp"], toy["be"]
    be.graph.params.reset()
    res = C.run_session(hp=hp, be=be, arrivals_ns=toy["arrivals"], log_capacity=1 << 22, hp_latency_ns=20_000)
    out_col = hp.out.clone()
    K = len(res["be_t_end"])
    p_col = be.graph.params.flat.cpu().clone()
    assert K >= 1
    # (1) bit-exact decision log vs the oracle replay of the recorded tape
    hdr, prefix, tape, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    kinds = {d[1] for d in lf.decode_decisions(decs)}
    assert 1 in kinds and kinds & {3, 4}
    # (2) HP outputs vs oracle
    P = toy["P"]
    worst = 0.0
    for r in range(hp.n_req):
        ref = om.mlp_fwd(P, toy["xs_hp"][r])
        worst = max(worst, rel(out_col[r].view(1, 512), ref))
    assert worst < 1e-4, worst
    # (3) BE parameters after K iterations vs oracle (cycling the 8 pre-staged batches)
    Po = dict(P)
    for i in range(K):
        _, Po, _ = om.mlp_train_step(Po, toy["xs_be"][i % 8], toy["ts_be"][i % 8], lr=0.01)
    flat_ref = torch.cat([Po[n].reshape(-1) for n, _, _ in W.mlp_spec()])
    assert rel(p_col, flat_ref) < 1e-4
    # (4) solo runs: bitwise identical outputs
    hp.out.zero_()
    C.run_session(hp=hp, arrivals_ns=toy["arrivals"])
    assert torch.equal(hp.out, out_col)
    be.graph.params.reset()
    C.run_session(be=be, be_iters=K)
    assert torch.equal(be.graph.params.flat.cpu(), p_col)


def test_toy_three_be_clients(toy):
    """one HP client and three BE training clients (each its own MLP,
    buffers and stream) share one DUR budget round robin. The decision log must equal the oracle
    replay byte for byte; every BE client's parameters after its K_j iterations must equal the
    fp64 oracle's and be bitwise identical to a solo run of that client."""
    hp = toy["hp"]
    P = toy["P"]
    bes = []
    for j in range(3):
        xs = [si.normal((32, 512), si.BE_SEED, sub=10 * (j + 1) + i) for i in range(2)]
        ts = [si.normal((32, 512), si.BE_SEED, sub=200 + 10 * (j + 1) + i) for i in range(2)]
        g = W.mlp_train_graph(P, xs, ts, lr=0.01)
        prof, _ = PR.build_profiles(g, kid_base=1000 * (j + 1), reps=3)
        g.params.reset()
        bes.append((C.BEClient(g, prof, 1000 * (j + 1)), xs, ts))
    res = C.run_session(hp=hp, be=[b for b, _, _ in bes], arrivals_ns=toy["arrivals"][:100], log_capacity=1 << 22,
                        hp_latency_ns=20_000)
    hdr, prefix, tape, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    clients = {d[2] for d in lf.decode_decisions(decs) if d[1] in (3, 4)}
    assert len(clients) == 3, clients          # every BE client was admitted
    for j, (b, xs, ts) in enumerate(bes):
        K = len(res["be_t_end_all"][j])
        assert K >= 1
        p_col = b.graph.params.flat.cpu().clone()
        Po = dict(P)
        for i in range(K):
            _, Po, _ = om.mlp_train_step(Po, xs[i % 2], ts[i % 2], lr=0.01)
        flat_ref = torch.cat([Po[n].reshape(-1) for n, _, _ in W.mlp_spec()])
        assert rel(p_col, flat_ref) < 1e-4
        b.graph.params.reset()
        C.run_session(be=b, be_iters=K)
        assert torch.equal(b.graph.params.flat.cpu(), p_col)


@pytest.mark.parametrize("policy", ["priorities", "profiles", "streams", "orion_noprio"])
def test_toy_policy_ablation_log(toy, policy):
    """The ablation switches (Fig. 14) on real kernels: the decision log of each
    policy variant equals the oracle replay of its own tape, and outputs stay bitwise identical to
    the default policy's solo run (scheduling never changes results)."""
    hp, be = toy["hp"], toy["be"]
    be.graph.params.reset()
    hp.out.zero_()
    res = C.run_session(hp=hp, be=be, arrivals_ns=toy["arrivals"][:60], log_capacity=1 << 22, hp_latency_ns=20_000,
                        flags=L.POLICIES[policy])
    hdr, prefix, tape, decs = lf.split_log(res["log"])
    assert decs == po.replay(prefix)
    kinds = {d[1] for d in lf.decode_decisions(decs)}
    if policy in ("priorities", "streams"):
        assert not kinds & {5, 6, 7, 8}, kinds      # no defers, no resets: every BE op admitted at once
    out_col = hp.out[:60].clone()
    hp.out.zero_()
    C.run_session(hp=hp, arrivals_ns=toy["arrivals"][:60])
    assert torch.equal(hp.out[:60], out_col)
