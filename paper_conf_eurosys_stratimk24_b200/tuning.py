"""SM_THRESHOLD tuning for a throughput-oriented (training) HP client (§5.1.1, P:617-620,
P:658-665): "Tuning is done by monitoring the throughput of the high-priority job and adjusting the
SM_THRESHOLD with binary search, using the maximum number of SMs needed by any kernel of the
best-effort job as the max value and zero as the min value in the search."

Reading R33: the search keeps the largest threshold whose measured HP throughput stays
at >= `keep` (0.8) of dedicated. The upper end is max BE sm_needed + 1, because the SM test is strict
(L27: sm_needed < SM_THRESHOLD), so only that value admits the largest BE kernel beside the HP;
threshold 0 admits nothing beside a busy HP (HP at its dedicated throughput). The search assumes
the HP fraction is non-increasing in the threshold (a larger threshold only admits more BE kernels).

The search itself is host logic (no GPU): `measure(threshold)` runs a collocated window -- on the
GPU in bench.py (config 4), on the FAKE backend's SM-contention model in the CPU tests.
"""


def search_sm_threshold(measure, max_sm_needed, keep=0.8, max_probes=7):
    """Binary search of SM_THRESHOLD over [0, max_sm_needed + 1].

    measure(thr) -> HP throughput as a fraction of dedicated. Returns (tuned, probes) with probes a
    list of (threshold, fraction) in probe order. The most aggressive threshold is probed first (if
    it keeps the HP, it is the answer); then the bracket [lo, hi) with fraction(lo) >= keep >
    fraction(hi) is halved until it is one apart or the probe budget is spent."""
    lo, hi = 0, int(max_sm_needed) + 1
    probes = []
    f = float(measure(hi))
    probes.append((hi, f))
    if f >= keep:
        return hi, probes
    while hi - lo > 1 and len(probes) < max_probes:
        mid = (lo + hi) // 2
        f = float(measure(mid))
        probes.append((mid, f))
        if f >= keep:
            lo = mid
        else:
            hi = mid
    return lo, probes


def fake_hp_fraction(hp_ops, be_ops, threshold, n_hp_iters=20, dedicated_s=None, dur_ns_hp=None):
    """One collocated window on the FAKE backend with its SM-contention model: a throughput-mode HP
    training client (n_hp_iters iterations of hp_ops submitted at once, as bench.py's train-train
    mode does: the HP is never idle) beside a closed-loop BE client (be_ops), at the given
    SM_THRESHOLD (>= 1; 0 means the default, #SMs). Returns the HP's iterations/s (and, if
    dedicated_s is given, the fraction of it)."""
    import ctypes
    import threading
    import time

    from . import _lib as L
    from .runtime import Orion

    o = Orion(backend=L.BACKEND_FAKE, sm_threshold=threshold, fake_contention=True, hp_latency_ns=dur_ns_hp or 0,
              dur_threshold_ppm=25000, queue_capacity=1024)
    hp = o.register_client(L.HP)
    be = o.register_client(L.BE) if be_ops else None
    o.start()
    stop = ctypes.c_int32(0)
    th = None
    if be is not None:
        th = threading.Thread(target=lambda: o.run_iterations(be, [be_ops], stop_flag=stop))
        th.start()
    t0 = time.perf_counter()
    for _ in range(n_hp_iters):
        for op in hp_ops:
            while o.submit(hp, op) is None:
                time.sleep(0)
    o.synchronize(hp)
    dt = time.perf_counter() - t0
    stop.value = 1
    if th is not None:
        th.join()
    o.stop()
    o.destroy()
    its = n_hp_iters / dt
    return its / dedicated_s if dedicated_s else its
