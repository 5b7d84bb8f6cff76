"""SM_THRESHOLD tuning for a throughput HP (reading R33): the binary search itself
against step-function throughput models (every answer checked by brute force), and end to end on
liborion's FAKE backend with its SM-contention model driving real scheduler sessions."""
import math

import pytest

import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import _lib as L, tuning as T


def brute(measure, max_sm, keep):
    """Largest threshold in [0, max_sm + 1] whose fraction is >= keep (0 if none; the model's
    fraction is non-increasing in the threshold)."""
    best = 0
    for t in range(1, max_sm + 2):
        if measure(t) >= keep:
            best = t
    return best


@pytest.mark.parametrize("max_sm,cut", [(148, 0), (148, 1), (148, 60), (148, 148), (148, 149), (296, 150),
                                        (7, 3), (1000, 999), (31, 16)])
def test_search_matches_brute_force_with_enough_probes(max_sm, cut):
    calls = []

    def measure(t):           # HP keeps 95 % up to `cut`, 60 % beyond (non-increasing)
        calls.append(t)
        return 0.95 if t <= cut else 0.6
    budget = 1 + math.ceil(math.log2(max_sm + 2))
    tuned, probes = T.search_sm_threshold(measure, max_sm, keep=0.8, max_probes=budget)
    assert tuned == brute(lambda t: 0.95 if t <= cut else 0.6, max_sm, 0.8)
    assert probes[0][0] == max_sm + 1          # the most aggressive threshold is probed first
    assert len(probes) <= budget and [p[0] for p in probes] == calls


def test_search_is_safe_when_the_budget_runs_out():
    """With fewer probes than log2(range) the answer is a threshold that was measured to keep the
    HP (a lower bound of the optimum), never an unmeasured one."""
    for cut in range(1, 300, 7):
        tuned, probes = T.search_sm_threshold(lambda t: 1.0 if t <= cut else 0.5, 300, keep=0.8, max_probes=4)
        assert tuned <= cut
        assert tuned == 0 or any(p[0] == tuned and p[1] >= 0.8 for p in probes)


def test_search_all_or_nothing():
    assert T.search_sm_threshold(lambda t: 1.0, 200)[0] == 201          # every BE kernel may run beside the HP
    tuned, probes = T.search_sm_threshold(lambda t: 0.1, 200, max_probes=20)
    assert tuned == 0 and len(probes) <= 1 + math.ceil(math.log2(202))


def _ops(spec, kid0):
    return [orion.make_op(0, [], kernel_id=kid0 + i, cls=c, sm_needed=s, dur_ns=d) for i, (c, s, d) in enumerate(spec)]


def test_search_on_fake_backend_contention_model():
    """HP: compute-bound kernels on 100 SMs; BE: memory-bound kernels of 30, 60 and 140 SMs. Beside
    the HP, 30 fits (130 <= 148), 60 over-subscribes a little (160: the HP runs at 148/160 while they
    overlap) and 140 a lot (240). With keep = 0.8 the search must stop right below the 140-SM
    kernel's admission (threshold 140: sm_needed < 140 admitted), matching brute force over the
    boundary thresholds measured on the same model."""
    hp_ops = _ops([(L.CLS_C, 100, 200_000)] * 10, 0)
    be_ops = _ops([(L.CLS_M, 30, 100_000), (L.CLS_M, 60, 150_000), (L.CLS_M, 140, 400_000)] * 2, 100)
    ded = T.fake_hp_fraction(hp_ops, None, 1)

    def measure(t):
        return T.fake_hp_fraction(hp_ops, be_ops, t, dedicated_s=ded)
    fr = {t: measure(t) for t in (31, 60, 61, 140, 141)}
    assert fr[31] > 0.95 and fr[60] > 0.95          # only the 30-SM kernel beside the HP: no contention
    assert 0.8 < fr[61] and fr[140] > 0.8            # the 60-SM kernel too: mild contention
    assert fr[141] < 0.75                            # the 140-SM kernel: the HP loses > 25 %
    tuned, probes = T.search_sm_threshold(measure, 140, keep=0.8, max_probes=10)
    assert tuned == 140, probes
    for t, f in probes:
        assert (f >= 0.8) == (t <= 140), probes
