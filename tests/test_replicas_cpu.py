"""The N>1 path on CPU: two gloo ranks, each an independent Orion instance (FAKE backend: CPU
threads as streams) running HP requests + BE iterations; the control plane gathers per-rank
numbers and aggregates them (sum of throughput, max of time) exactly as bench.py does."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_main(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    import ctypes
    import threading
    import numpy as np
    import paper_conf_eurosys_stratimk24_b200 as orion
    from paper_conf_eurosys_stratimk24_b200 import _lib as L, replicas as R
    r, w, local = R.init_from_env()
    o = orion.Orion(backend=L.BACKEND_FAKE, hp_latency_ns=200_000, log_capacity=1 << 16)
    hp, be = o.register_client(L.HP), o.register_client(L.BE)
    o.start()
    hp_ops = [orion.make_op(0, [], kernel_id=i, cls=1, sm_needed=10, dur_ns=20_000 * (rank + 1)) for i in range(4)]
    be_ops = [[orion.make_op(0, [], kernel_id=100 + i, cls=2, sm_needed=10, dur_ns=30_000) for i in range(6)]]
    stop = ctypes.c_int32(0)
    res = {}
    R.barrier()
    t = threading.Thread(target=lambda: res.setdefault("be", o.run_iterations(be, be_ops, stop)))
    t.start()
    ta, td = o.run_requests(hp, hp_ops, (np.arange(1, 11) * 1_000_000 * (rank + 1)).astype(np.int64))
    stop.value = 1
    t.join()
    o.stop()
    o.destroy()
    lat = np.sort(td - ta)
    mine = dict(be_col=float(len(res["be"])), be_ded=1.0, win_ms=10.0 * (rank + 1), p99=float(lat[-1]), p99d=float(lat[0]),
                p50=0.0, p50d=0.0, be_n=len(res["be"]))
    allr = R.gather(mine)
    if r == 0:
        q.put((allr, R.aggregate(allr, steps=10)))
    R.barrier()


def test_two_gloo_replicas_aggregate():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(i, 2, port, q)) for i in range(2)]
    for p in procs:
        p.start()
    allr, agg = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert len(allr) == 2 and allr[0]["win_ms"] == 10.0 and allr[1]["win_ms"] == 20.0
    assert agg["value"] == allr[0]["be_col"] + allr[1]["be_col"]
    assert agg["ms_per_step"] == 2.0
    assert agg["hp_p99_ratio_max"] == max(r["p99"] / r["p99d"] for r in allr)
