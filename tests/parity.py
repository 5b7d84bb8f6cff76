"""Parity measures shared by the GPU tests (DESIGN.md §8 states the error model behind each).

  rel(got, ref)            per-tensor relative L2 (R23)
  elem(got, ref)           max |got - ref| / rms(ref): the elementwise companion of rel. For rounding
                           noise spread over n elements the max is ~sqrt(2 ln n) (<= ~6.5 for
                           n <= 1e9) times the rms error, so ELEM_FACTOR x the rel tolerance holds for
                           an honest result; a localized tile / tail error fails it long before it
                           moves the per-tensor norm
  cond_elem(got, ref, A)   max_e |got - ref|_e / A_e with A_e the absolute-term sum of element e
                           (Higham: |fl(sum t) - sum t| <= gamma sum |t|): the bound that holds for a
                           reduction whose terms cancel (BN parameter gradients, weight gradients)
  kappa(ref, A)            ||A|| / ||ref||: the cancellation ratio, the factor by which the relative
                           error of a cancelling reduction legitimately exceeds its inputs'
  audit_decisions(...)     the ReLU / ReLU6 pass/stop decisions the GPU took against the oracle's own
"""
import math

import torch

ELEM_FACTOR = 10.0


def _dd(t):
    return torch.as_tensor(t).detach().double().cpu()


def rel(got, ref, floor=1e-30):
    a, b = _dd(got), _dd(ref)
    return float((a - b).norm() / max(float(b.norm()), floor))


def elem(got, ref, floor=1e-30):
    a, b = _dd(got), _dd(ref)
    rms = float(b.norm()) / math.sqrt(max(b.numel(), 1))
    return float((a - b).abs().max()) / max(rms, floor) if b.numel() else 0.0


def cond_elem(got, ref, A, floor=1e-30):
    a, b, s = _dd(got), _dd(ref), _dd(A)
    return float(((a - b).abs() / s.clamp_min(floor)).max())


def kappa(ref, A):
    return float(_dd(A).norm()) / max(float(_dd(ref).norm()), 1e-300)


def assert_close(name, got, ref, rel_tol, elem_factor=ELEM_FACTOR, floor=1e-30):
    r, e = rel(got, ref, floor), elem(got, ref, floor)
    assert r <= rel_tol, f"{name}: rel L2 {r:.3e} > {rel_tol:.1e}"
    assert e <= elem_factor * rel_tol, f"{name}: max |err| / rms {e:.3e} > {elem_factor * rel_tol:.1e}"
    return r, e


def audit_decisions(name, y_gpu, y_oracle, thresholds=(0.0, 6.0), max_flip_frac=1e-4, rel_floor=5e-6):
    """The GPU's ReLU6 (thresholds 0, 6) or ReLU (0) decided on y_gpu; the oracle's own free-running
    forward produced y_oracle. Measures the forward drift of this tensor (rel L2, max |err| / rms) and
    checks:
      * the drift is spread like rounding noise, not localized: max |err| <= ELEM_FACTOR x
        max(rel, rel_floor) x rms (a wrong tile or row has a max far above its share of the norm;
        rel_floor = 5e-6 ~ 80 u absorbs BN's per-channel amplification of a few-ulp error, five
        orders of magnitude below the O(rms) error of a wrong index);
      * every element where the two take different decisions has its oracle value within that band
        of a threshold, and flips are rare (<= max(max_flip_frac, 2 rel) of the elements).
    Returns (flips, rel). The caller checks that the drift grows smoothly along the forward pass."""
    g, o = _dd(y_gpu).reshape(-1), _dd(y_oracle).reshape(-1)
    rms = float(o.norm()) / math.sqrt(max(o.numel(), 1))
    r = float((g - o).norm() / max(float(o.norm()), 1e-30))
    delta = ELEM_FACTOR * max(r, rel_floor) * rms
    err = float((g - o).abs().max())
    assert err <= delta, f"{name}: forward max |err| {err:.3e} > {ELEM_FACTOR:g} x rel {r:.2e} x rms (localized error?)"
    lo = thresholds[0]
    if len(thresholds) == 2:
        hi = thresholds[1]
        dg, do = (g > lo) & (g < hi), (o > lo) & (o < hi)
        near = torch.minimum((o - lo).abs(), (o - hi).abs())
    else:
        dg, do = g > lo, o > lo
        near = (o - lo).abs()
    flip = dg != do
    nflip = int(flip.sum())
    if nflip:
        worst = float(near[flip].max())
        assert worst <= delta, f"{name}: decision flip at an oracle value {worst:.3e} from a threshold (band {delta:.3e})"
        # a flip needs |o - t| < |g - o|: P(flip) ~ 2 f(t) E|g - o| <= 2 (0.5 / rms) (r rms) = r for a
        # value density f(t) <= 0.5 / rms at the threshold (a unit-variance normal peaks at 0.40)
        cap = max(1, max_flip_frac * o.numel(), 2.0 * r * o.numel())
        assert nflip <= cap, f"{name}: {nflip} decision flips of {o.numel()} (cap {cap:.0f})"
    return nflip, r


def check_train_iterations(run_one, graph, step, xs, labels, P0, K, dec_attr, thresholds, audit_skip=(), tau_g=1e-4,
                           lr=0.01, mu=0.9, trace_order="forward", drift_floor=1e-4, drift_jump=2.0):
    """K training iterations on the GPU vs the fp64 oracle with audited decisions.

    run_one(it): runs GPU iteration `it` (batch it) from the graph's current parameters.
    step(P, V, x, labels, first, masks, trace) -> (loss, newP, newV, grads): the oracle step.
    dec_attr: the graph's dict of the values its ReLU / ReLU6 backward decided on (name -> tensor);
    the oracle's trace key of the same values is "bn_out" or "relu_in"; names with a suffix in
    audit_skip feed no activation and are not audited.
    Per iteration: decisions audited (audit_decisions: drift spread like noise, flips only inside
    the drift band and rare) and the drift must grow smoothly along the forward pass (each tensor's
    rel L2 <= max(drift_floor, drift_jump x the largest drift before it): the fp32 forward drifts
    geometrically through a deep train-mode network, ~8 % per ResNet block, while a wrong kernel shows
    as a jump); trace_order says whether the oracle's trace lists the tensors in forward or backward
    order; loss rel 1e-5; every gradient element within tau of its absolute-term sum, every
    gradient tensor within tau x max(1, kappa) in rel L2, tau = tau_g + 2 x the iteration's worst
    forward drift (the operands' perturbation a gradient inherits). After K: momentum (accumulated sums)
    and parameters (K ulps of storage rounding per side + lr x the accumulated bound); BN running
    statistics rel 1e-5 + 2 x the worst forward drift (rmean with an absolute floor of 1e-2: block outputs have exactly zero
    batch mean, so their next BN's running mean is rounding noise). Returns a per-iteration report."""
    G = graph.params
    base = G.gflat.data_ptr()
    V_gpu = {n: G.vflat[(t.data_ptr() - base) // 4:(t.data_ptr() - base) // 4 + t.numel()].view(t.shape) for n, t in G.g.items()}
    Po, Vo = dict(P0), {}
    A_v, A_vsum, report, tau_acc, drift_acc = {}, {}, [], tau_g, 0.0
    for it in range(K):
        run_one(it)
        masks = {k: v.cpu() for k, v in getattr(graph, dec_attr).items()}
        tr = {}
        loss_o, newP, newV, g_o = step(Po, Vo, xs[it], labels[it], it == 0, masks, tr)
        own = tr.get("bn_out", tr.get("relu_in"))
        names = [n for n in own if n in masks and not n.endswith(tuple(audit_skip))]
        if trace_order == "backward":
            names = names[::-1]
        flips, run_max, worst_drift, drifts = 0, 0.0, 0.0, []
        for name in names:
            f, r = audit_decisions(f"iter {it} {name}", masks[name], own[name], thresholds)
            assert r <= max(drift_floor, drift_jump * run_max), f"iter {it} {name}: forward drift {r:.2e} jumps over {run_max:.2e}"
            run_max = max(run_max, r)
            drifts.append((name, r))
            worst_drift = max(worst_drift, r)
            flips += f
        lr_ = rel(graph.loss, loss_o.reshape(1))
        print(" ".join(f"{n}:{r:.1e}" for n, r in drifts[:: max(1, len(drifts) // 24)]), flush=True)
        print(f"iter {it}: loss rel {lr_:.3e}, flips {flips}, worst forward drift {worst_drift:.3e}", flush=True)
        assert lr_ < 1e-5, f"iter {it}: loss rel {lr_:.3e}"
        # a gradient g = sum a b inherits its operands' relative perturbation: |dg| <= sum |a||b| (|da/a| +
        # |db/b|) + gamma sum |a||b|, so its bound is tau_g plus the forward drift of both operands
        tau_it = tau_g + 2.0 * worst_drift
        tau_acc = max(tau_acc, tau_it)
        drift_acc = max(drift_acc, worst_drift)
        worst_c, worst_r, worst_k = 0.0, 0.0, 0.0
        for n, ref in g_o.items():
            A = tr["abs"][n]
            ce, k, r = cond_elem(G.g[n], ref, A), kappa(ref, A), rel(G.g[n], ref)
            assert ce <= tau_it, f"iter {it} {n}: max |err| / abs-sum {ce:.3e} > {tau_it:.3g}"
            if k < 1e6:   # exactly-zero true gradients are held by the elementwise bound only
                assert r <= tau_it * max(1.0, k), f"iter {it} {n}: rel {r:.3e} > {tau_it:.3g} x kappa {k:.1f}"
                worst_r = max(worst_r, r)
                worst_k = max(worst_k, k)
            worst_c = max(worst_c, ce)
            A_v[n] = A.double() if it == 0 else mu * A_v[n] + A.double()
            A_vsum[n] = A_v[n] if it == 0 else A_vsum[n] + A_v[n]
        report.append(dict(iter=it, loss=float(loss_o), flips=flips, worst_forward_drift=worst_drift, grad_tol=tau_it,
                           worst_cond_elem=worst_c, worst_rel=worst_r, worst_kappa=worst_k))
        Po, Vo = newP, newV
    for n, ref in Vo.items():
        ce = cond_elem(V_gpu[n], ref, A_v[n])
        assert ce <= tau_acc, f"momentum {n}: {ce:.3e}"
    for n, ref in Po.items():
        p, r = _dd(G.p[n]), _dd(ref)
        if n in A_vsum:
            bound = 2 * K * (2.0 ** -23) * r.abs() + tau_acc * lr * A_vsum[n] + 1e-30
            worst = float(((p - r).abs() / bound).max())
            assert worst <= 1.0, f"param {n}: {worst:.3f} x (storage rounding + lr x gradient bound)"
        else:
            # running statistics are batch statistics of drifted activations: 1e-5 + 2 x the drift
            tol = 1e-5 + 2.0 * drift_acc
            assert rel(p, r, 1e-2 if n.endswith(".rmean") else 1e-30) < tol, f"{n}: rel {rel(p, r):.3e} > {tol:.3e}"
    return report
