"""Pins for the policy oracle (oracle/policy.c): hand-derived worked examples + brute force.

WE1-WE6 (tests/golden/we*.txt) are derived by hand from Listing 1 and the
readings of DESIGN.md §3; the brute force checks invariants I1-I11, which
restate the paper's prose: HP launched at once on its stream, BE admission rule
(P:603-618), throttle, FIFO per client, unknown optimism.
"""
import glob
import itertools
import os
import random

import pytest

from oracle import policy_ffi as po
import logfmt as lf

GOLD = os.path.join(os.path.dirname(__file__), "golden")


@pytest.mark.parametrize("path", sorted(glob.glob(os.path.join(GOLD, "we*.txt"))))
def test_worked_example(path):
    log, expect = lf.parse_golden(path)
    got = lf.decode_decisions(po.replay(log))
    assert got == expect, (os.path.basename(path), got)


def _mk(ops_per_client, prios, dur_thr=10000, flags=0, num_sms=148, sm_thr=148):
    return lf.encode(num_sms, sm_thr, dur_thr, flags, prios, ops_per_client, tape=None)


def _op(kid, cls, sm, dur, kind=0, opf=0):
    return (kid, kind, opf, cls, sm, dur)


ALL_FLAGS = [0, 1, 2, 4, 8, 16, 1 | 2, 2 | 16, 4 | 8, 31, 64, 128, 256, 64 | 128 | 256, 32 | 64 | 128 | 256, 128 | 2]


@pytest.mark.parametrize("flags", ALL_FLAGS)
def test_brute_hp2_be3(flags):
    """Every tape of HP=2 ops + 1 BE client with 3 ops, profiles spanning the decision edges."""
    hp = [_op(1, 1, 40, 50000), _op(2, 2, 147, 30000)]
    be = [_op(10, 2, 20, 9999), _op(11, 1, 148, 10000), _op(12, 0, 1, 10001)]
    r, paths, nodes, err = po.brute(_mk([hp, be], [0, 1], flags=flags))
    assert r == 0, err
    assert paths > 1000


@pytest.mark.parametrize("flags", [0, 2, 8, 16])
def test_brute_two_be_clients(flags):
    hp = [_op(1, 2, 20, 30000)]
    a = [_op(10, 2, 10, 8000), _op(11, 1, 200, 2000)]
    b = [_op(20, 0, 4, 10001), _op(21, 1, 147, 0, kind=1)]   # memop second
    r, paths, nodes, err = po.brute(_mk([hp, a, b], [0, 1, 1], flags=flags), max_nodes=3_000_000)
    assert r == 0, err
    assert paths > 100


def test_brute_request_flags():
    """HP_BUSY_REQUEST: request boundaries via REQ_BEGIN/REQ_END op flags."""
    hp = [_op(1, 1, 40, 100, opf=1), _op(2, 2, 40, 100, opf=2), _op(3, 0, 8, 100, opf=3)]
    be = [_op(10, 2, 20, 5000), _op(11, 1, 20, 5000)]
    r, paths, nodes, err = po.brute(_mk([hp, be], [0, 1], flags=1 | 2))
    assert r == 0, err


def test_brute_detects_broken_threshold():
    """Sanity of the checker itself: with dur_thr so large nothing throttles, I5/I6 still hold;
    an inconsistent header (BE op dur larger than thr + max) can't exist, so instead verify the
    brute force actually explores (non-trivial path counts)."""
    be = [_op(10, 2, 20, 5), _op(11, 1, 20, 5)]
    r, paths, nodes, err = po.brute(_mk([be], [1], dur_thr=0))
    assert r == 0 and paths >= 3 and nodes > paths


def _random_trace(rng, n_hp, n_be_clients, n_be):
    prios = ([0] if n_hp else []) + [1] * n_be_clients
    ops = []
    if n_hp:
        ops.append([_op(rng.randrange(1, 50), rng.choice([0, 1, 2]), rng.choice([1, 40, 147, 148, 200]),
                        rng.choice([0, 9999, 10000, 10001, 50000])) for _ in range(n_hp)])
    for _ in range(n_be_clients):
        ops.append([_op(rng.randrange(50, 100), rng.choice([0, 1, 2]), rng.choice([1, 40, 147, 148, 200]),
                        rng.choice([0, 9999, 10000, 10001, 50000]),
                        kind=(1 if rng.random() < 0.15 else 0)) for _ in range(n_be)])
    return prios, ops


def test_brute_random_fuzz():
    rng = random.Random(1234)
    for it in range(40):
        prios, ops = _random_trace(rng, rng.choice([0, 1, 2]), rng.choice([1, 2]), rng.choice([1, 2]))
        flags = rng.choice(ALL_FLAGS)
        r, paths, nodes, err = po.brute(_mk(ops, prios, flags=flags), max_nodes=400_000)
        assert r == 0, (it, flags, err)


def test_replay_deterministic_and_quiescence_exact():
    """I9: replay of the same tape twice is identical; the quiescence jump is exact: stretching
    every gap between tape stamps by a multiple of n_be changes only the k of the records."""
    log, expect = lf.parse_golden(os.path.join(GOLD, "we5.txt"))
    a = po.replay(log)
    assert a == po.replay(log)
    hdr, _ = lf.decode_header(log)
    # WE1 with stamps scaled by 10: decisions at the stamp iterations move, the sequence stays.
    log1, exp1 = lf.parse_golden(os.path.join(GOLD, "we1.txt"))
    h1, off = lf.decode_header(log1)
    tape = [(0, 1, 0, 3), (300, 2, 0, 1), (570, 2, 0, 2)]
    log2 = lf.encode(148, 148, 10000, 0, h1["prios"], h1["ops"], tape, k_end=1000)
    got = lf.decode_decisions(po.replay(log2))
    assert [g[1:] for g in got] == [e[1:] for e in exp1]
    assert [g[0] for g in got] == [0, 1, 2, 570, 570]


def test_k_end_truncates():
    log, expect = lf.parse_golden(os.path.join(GOLD, "we1.txt"))
    hdr, off = lf.decode_header(log)
    _, _, tape, _ = lf.split_log(log + b"")
    log2 = lf.encode(148, 148, 10000, 0, hdr["prios"], hdr["ops"], tape, k_end=40)
    got = lf.decode_decisions(po.replay(log2))
    assert got == expect[:3]


MUTANTS = {1: "SM test <= instead of <", 2: "profile test inverted", 3: "unknown treated as its own class",
           4: "DUR test >= instead of >", 5: "reset without drain", 6: "be_dur not accumulated",
           7: "hp_busy never set", 8: "no BE round-robin rotation",
           9: "HP_REF_ALL checks only the newest in-flight HP op",
           10: "HP_BUSY_REQUEST ignores a request whose last op is not popped yet"}


@pytest.mark.parametrize("m", sorted(MUTANTS))
def test_pins_catch_mutant(m, tmp_path):
    """Each plausible mistake in the policy must fail a golden example or the brute force."""
    import ctypes
    import subprocess
    so = str(tmp_path / f"mut{m}.so")
    subprocess.check_call(["gcc", "-O1", "-std=c11", "-fPIC", "-shared", f"-DORACLE_MUTANT={m}", "-o", so,
                           os.path.join(po.ORACLE_DIR, "policy.c")])
    L = ctypes.CDLL(so)
    L.oracle_replay.argtypes = po.lib().oracle_replay.argtypes
    L.oracle_brute.argtypes = po.lib().oracle_brute.argtypes
    caught = []
    for path in sorted(glob.glob(os.path.join(GOLD, "we*.txt"))):
        log, expect = lf.parse_golden(path)
        need = ctypes.c_size_t(0)
        buf = ctypes.create_string_buffer(1 << 16)
        r = L.oracle_replay(log, len(log), buf, 1 << 16, ctypes.byref(need))
        if r != 0 or lf.decode_decisions(buf.raw[:need.value]) != expect:
            caught.append(os.path.basename(path))
    hp = [_op(1, 1, 40, 50000), _op(2, 2, 147, 30000)]
    be = [_op(10, 2, 20, 9999), _op(11, 1, 148, 10000), _op(12, 0, 1, 10001)]
    hdr = _mk([hp, be], [0, 1])
    paths, nodes = ctypes.c_uint64(0), ctypes.c_uint64(0)
    err = ctypes.create_string_buffer(256)
    if L.oracle_brute(hdr, len(hdr), 0, ctypes.byref(paths), ctypes.byref(nodes), err, 256) != 0:
        caught.append("brute:" + err.value.decode())
    assert caught, f"mutant {m} ({MUTANTS[m]}) not caught by any pin"
