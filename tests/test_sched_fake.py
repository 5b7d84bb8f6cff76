"""liborion's scheduler on the FAKE backend (CPU threads play the streams): the decision log the
library writes must equal, byte for byte, the oracle's replay of the library's own observation tape
(the bit-exactness contract of BASELINE.json north_star). No GPU needed."""
import random
import threading
import time

import pytest

import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import _lib as L
from oracle import policy_ffi as po
import logfmt as lf


def _rand_ops(rng, n, kid0):
    ops = []
    for i in range(n):
        mem = rng.random() < 0.08
        ops.append(orion.make_op(0, [], kernel_id=kid0 + i, cls=rng.choice([0, 1, 2]),
                                 sm_needed=rng.choice([1, 8, 40, 147, 148, 300]),
                                 dur_ns=rng.choice([0, 2000, 5000, 20000, 60000]),
                                 kind=L.OP_MEMCPY_H2D if mem else L.OP_KERNEL))
    return ops


def _producer(o, cid, ops, rng, burst):
    i = 0
    while i < len(ops):
        n = min(len(ops) - i, rng.randint(1, burst))
        for op in ops[i:i + n]:
            while o.submit(cid, op) is None:
                time.sleep(0)
        i += n
        time.sleep(rng.random() * 2e-4)


@pytest.mark.parametrize("seed,flags,n_be", [(1, 0, 1), (2, 0, 2), (3, L.F_HP_BUSY_REQUEST | L.F_HP_REF_ALL, 1),
                                             (4, L.F_FREE_SMS, 2), (5, L.F_HP_UNKNOWN_STRICT | L.F_THROTTLE_ONLY_HP_BUSY, 1),
                                             (6, 31, 3), (7, L.POLICIES["priorities"], 2), (8, L.POLICIES["profiles"], 1),
                                             (9, L.POLICIES["streams"], 2)])
def test_fake_log_matches_oracle(seed, flags, n_be):
    rng = random.Random(seed)
    o = orion.Orion(backend=L.BACKEND_FAKE, hp_latency_ns=1_000_000, dur_threshold_ppm=25000, flags=flags,
                    log_capacity=1 << 20, fake_time_scale_pct=100, queue_capacity=64)
    hp = o.register_client(L.HP)
    bes = [o.register_client(L.BE) for _ in range(n_be)]
    hp_ops = _rand_ops(rng, 120, 1000)
    for i, op in enumerate(hp_ops):           # request structure for HP_BUSY_REQUEST
        op.opflags = (L.OPF_REQ_BEGIN if i % 10 == 0 else 0) | (L.OPF_REQ_END if i % 10 == 9 else 0)
    be_ops = [_rand_ops(rng, 200, 5000 + 1000 * j) for j in range(n_be)]
    o.start()
    ths = [threading.Thread(target=_producer, args=(o, hp, hp_ops, random.Random(seed + 10), 10))]
    ths += [threading.Thread(target=_producer, args=(o, b, be_ops[j], random.Random(seed + 20 + j), 30))
            for j, b in enumerate(bes)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    o.stop()
    log = o.read_log()
    st = o.stats()
    o.destroy()
    hdr, prefix, tape, decs = lf.split_log(log)
    assert hdr["k_end"] == st["iterations"]
    assert [len(x) for x in hdr["ops"]] == [120] + [200] * n_be
    ref = po.replay(prefix)
    got, want = lf.decode_decisions(decs), lf.decode_decisions(ref)
    for i, (g, w) in enumerate(zip(got, want)):
        assert g == w, (i, g, w)
    assert decs == ref
    kinds = {d[1] for d in got}
    assert 1 in kinds and (3 in kinds or 4 in kinds)


def test_lifecycle_errors():
    o = orion.Orion(backend=L.BACKEND_FAKE)
    hp = o.register_client(L.HP)
    with pytest.raises(L.OrionError):
        o.register_client(L.HP)               # at most one HP client
    with pytest.raises(L.OrionError) as e:
        o.stop()                              # not started
    assert e.value.code == L.E_STATE
    o.start()
    with pytest.raises(L.OrionError) as e:
        o.register_client(L.BE)               # registration after start
    assert e.value.code == L.E_STATE
    o.stop()
    with pytest.raises(L.OrionError) as e:
        o.read_log()                          # logging disabled
    o.destroy()


def test_queue_full_again():
    o = orion.Orion(backend=L.BACKEND_FAKE, queue_capacity=4)
    be = o.register_client(L.BE)
    op = orion.make_op(0, [], dur_ns=10_000_000)
    seqs = [o.submit(be, op) for _ in range(5)]   # not started: nothing drains
    assert seqs[:4] == [0, 1, 2, 3] and seqs[4] is None
    o.start()
    o.synchronize(be, timeout_ns=5_000_000_000)
    assert o.done_seq(be) == 4
    o.stop()
    o.destroy()


def test_native_drivers_fake():
    """orion_run_requests (open loop) and orion_run_iterations (closed loop) on the FAKE backend."""
    import ctypes
    import numpy as np
    o = orion.Orion(backend=L.BACKEND_FAKE, hp_latency_ns=100_000)
    hp = o.register_client(L.HP)
    be = o.register_client(L.BE)
    o.start()
    hp_ops = [orion.make_op(0, [], kernel_id=i, cls=1, sm_needed=10, dur_ns=20_000) for i in range(5)]
    be_ops = [[orion.make_op(0, [], kernel_id=100 + i, cls=2, sm_needed=10, dur_ns=30_000) for i in range(8)]]
    stop = ctypes.c_int32(0)
    res = {}
    t = threading.Thread(target=lambda: res.setdefault("be", o.run_iterations(be, be_ops, stop)))
    t.start()
    arr = np.arange(1, 21, dtype=np.int64) * 2_000_000
    ta, td = o.run_requests(hp, hp_ops, arr)
    stop.value = 1
    t.join()
    o.stop()
    lat = td - ta
    assert (lat > 100_000).all() and (lat < 50_000_000).all()
    assert len(res["be"]) > 5
    o.destroy()
