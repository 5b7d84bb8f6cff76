"""Collocation sessions: one Orion instance, one HP client (open-loop inference requests) and BE
clients (closed-loop training iterations), driven by liborion's native client drivers
(orion_run_requests / orion_run_iterations) so no Python sits between the clients and the
scheduler (P:1082-1085 notes Python client threads contend on the GIL).

Dedicated runs (the "Ideal" baseline) use the same binary with the other client
absent (R20).
"""
import ctypes
import os
import threading

import numpy as np
import torch

from . import _lib as L
from .runtime import Orion


class HPClient:
    """Inference client: graph with an H2D input memop first and a D2H output memop last."""

    def __init__(self, graph, inputs_host, n_req, profiles=None, kid_base=0):
        self.graph = graph
        self.n_req = n_req
        in_elems = graph.ops[0][1][2] // 4
        out_elems = graph.ops[-1][1][2] // 4
        self.inp = torch.empty((len(inputs_host), in_elems), dtype=torch.float32).pin_memory()
        for i, x in enumerate(inputs_host):
            self.inp[i].copy_(x.reshape(-1))
        self.out = torch.zeros((n_req, out_elems), dtype=torch.float32).pin_memory()
        self.set_profiles(profiles, kid_base)

    def set_profiles(self, profiles, kid_base=0):
        ops = self.graph.orion_ops(profiles, kid_base)
        ops[0].args[1] = self.inp.data_ptr()      # H2D src: request r uses input r % in_cycle
        ops[-1].args[0] = self.out.data_ptr()     # D2H dst: request r writes row r
        self.ops = ops


class BEClient:
    """Training client: op-list variants (one per pre-staged batch), run closed loop."""

    def __init__(self, graph, profiles=None, kid_base=0):
        self.graph = graph
        self.set_profiles(profiles, kid_base)

    def set_profiles(self, profiles, kid_base=0):
        self.variants = []
        for v in self.graph.variants:
            self.graph.ops = v
            self.variants.append(self.graph.orion_ops(profiles, kid_base))
        self.graph.ops = self.graph.variants[0]


def run_session(hp=None, be=None, arrivals_ns=None, be_iters=0, log_capacity=0, hp_latency_ns=0,
                dur_threshold_ppm=25000, sm_threshold=0, be_partition_sms=0, flags=0, sched_cpu=-1,
                backend=L.BACKEND_CUDA, device=0, trace_kernel_id=None, hp_cpu=None, be_cpus=None):
    """Run one session. HP (if given) issues len(arrivals_ns) requests open loop; BE (a client or a
    list of clients, each on its own thread and stream) runs closed loop until HP finishes (or
    be_iters iterations if HP is absent / be_iters > 0 and no HP).
    hp_cpu / be_cpus: host cores the HP driver (this thread, for the session) and the BE driver
    threads pin themselves to (placement.py), so no two busy-polling threads share a core.
    Returns dict with HP arrival/completion ns, BE iteration end times, window, log bytes, stats."""
    o = Orion(device=device, backend=backend, hp_latency_ns=hp_latency_ns, dur_threshold_ppm=dur_threshold_ppm,
              sm_threshold=sm_threshold, be_partition_sms=be_partition_sms, flags=flags, sched_cpu=sched_cpu,
              log_capacity=log_capacity, trace_kernel_id=trace_kernel_id)
    # several BE clients (R11: one shared DUR budget, round robin) when `be` is a list
    bes = [] if be is None else (list(be) if isinstance(be, (list, tuple)) else [be])
    hp_id = o.register_client(L.HP) if hp is not None else None
    be_ids = [o.register_client(L.BE) for _ in bes]
    torch.cuda.synchronize()
    o.start()
    res = {}
    stop = ctypes.c_int32(0)
    ths = []
    if bes:
        max_iters = be_iters if (hp is None or be_iters) else 0
        res["be_t_end_all"] = [None] * len(bes)

        def be_main(j):
            if be_cpus:
                os.sched_setaffinity(0, {be_cpus[j % len(be_cpus)]})
            try:
                res["be_t_end_all"][j] = o.run_iterations(be_ids[j], bes[j].variants, stop_flag=stop, max_iters=max_iters)
            except Exception as e:  # surfaced below
                res["be_err"] = e
        ths = [threading.Thread(target=be_main, args=(j,)) for j in range(len(bes))]
        res["t0"] = o_now = L.lib.orion_now_ns()
        for th in ths:
            th.start()
    else:
        res["t0"] = o_now = L.lib.orion_now_ns()
    prev_mask = os.sched_getaffinity(0) if hp_cpu is not None else None
    try:
        if hp is not None:
            if hp_cpu is not None:
                os.sched_setaffinity(0, {hp_cpu})
            ta, td = o.run_requests(hp_id, hp.ops, arrivals_ns, in_cycle=hp.inp.shape[0], out_cycle=hp.n_req)
            res["t_arrival"], res["t_done"] = ta, td
            res["t_hp_end"] = L.lib.orion_now_ns()
    except BaseException:
        # an HP driver error must not leave the BE threads spinning in native code: stop them,
        # join them and tear the instance down before the error propagates
        stop.value = 1
        for th in ths:
            th.join()
        try:
            o.stop()
        except Exception:
            pass
        o.destroy()
        raise
    finally:
        if prev_mask is not None:
            os.sched_setaffinity(0, prev_mask)
    if hp is not None:
        stop.value = 1
    for th in ths:
        th.join()
    if "be_err" in res:
        o.stop()
        o.destroy()
        raise res["be_err"]
    if bes:
        res["be_t_end"] = res["be_t_end_all"][0]
    res["t1"] = L.lib.orion_now_ns()
    o.stop()
    res["stats"] = o.stats()
    if trace_kernel_id is not None:
        res["trace_ms"] = o.trace_read()
    if log_capacity:
        res["log"] = o.read_log()
    o.destroy()
    del o_now
    return res


def run_direct(hp, arrivals_ns, device=0, hp_cpu=None):
    """The native arm (R20; P:1355-1360 measures Orion's overhead against it): the HP request stream
    launched directly on one stream by the client thread, no scheduler. Same completion counters and
    clock as run_session, so latencies compare one to one."""
    o = Orion(device=device, backend=L.BACKEND_CUDA)
    prev = os.sched_getaffinity(0)
    try:
        cid = o.register_client(L.HP)
        torch.cuda.synchronize()
        if hp_cpu is not None:
            os.sched_setaffinity(0, {hp_cpu})
        ta, td = o.run_requests_direct(cid, hp.ops, arrivals_ns, in_cycle=hp.inp.shape[0], out_cycle=hp.n_req)
    finally:
        os.sched_setaffinity(0, prev)
        o.destroy()
    return {"t_arrival": ta, "t_done": td}


def latency_stats(res):
    lat = (res["t_done"] - res["t_arrival"]).astype(np.float64)
    s = np.sort(lat)
    n = len(s)

    def pct(p):   # nearest rank (R19)
        return float(s[max(0, int(np.ceil(p / 100.0 * n)) - 1)])
    return dict(n=n, p50_ns=pct(50), p95_ns=pct(95), p99_ns=pct(99), mean_ns=float(lat.mean()))


def be_throughput(res, t_from=None, t_to=None):
    """BE iterations completed inside [t_from, t_to] per second (SURVEY §8(d) BE throughput)."""
    t = res.get("be_t_end", np.zeros(0, dtype=np.int64))
    t_from = res["t0"] if t_from is None else t_from
    t_to = res["t1"] if t_to is None else t_to
    n = int(((t >= t_from) & (t <= t_to)).sum())
    return n / ((t_to - t_from) / 1e9), n


def run_inference_session(hp=None, hp_arrivals=None, bes=(), be_arrivals=(), log_capacity=0, hp_latency_ns=0,
                          dur_threshold_ppm=25000, sm_threshold=0, be_partition_sms=0, flags=0, sched_cpu=-1,
                          backend=L.BACKEND_CUDA, device=0, hp_cpu=None, be_cpus=None):
    """Inf-inf session (Fig. 13): one HP and several BE *inference* clients, every one
    open loop with its own arrival trace, each driven by orion_run_requests on its own thread
    (BE requests go through Listing 1's BE path like any BE op; R11 rotates the BE clients). Any
    client may be absent (the dedicated runs). Returns {"hp": (t_arrival, t_done) or None,
    "be": [(t_arrival, t_done), ...], "t0", "t1", "stats", "log"}."""
    o = Orion(device=device, backend=backend, hp_latency_ns=hp_latency_ns, dur_threshold_ppm=dur_threshold_ppm,
              sm_threshold=sm_threshold, be_partition_sms=be_partition_sms, flags=flags, sched_cpu=sched_cpu,
              log_capacity=log_capacity)
    try:
        hp_id = o.register_client(L.HP) if hp is not None else None
        be_ids = [o.register_client(L.BE) for _ in bes]
        torch.cuda.synchronize()
        o.start()
    except BaseException:
        o.destroy()
        raise
    res = {"hp": None, "be": [None] * len(bes)}
    errs = []

    def be_main(j):
        if be_cpus:
            os.sched_setaffinity(0, {be_cpus[j % len(be_cpus)]})
        try:
            c = bes[j]
            res["be"][j] = o.run_requests(be_ids[j], c.ops, be_arrivals[j], in_cycle=c.inp.shape[0], out_cycle=c.n_req)
        except Exception as e:   # surfaced below
            errs.append(e)
    ths = [threading.Thread(target=be_main, args=(j,)) for j in range(len(bes))]
    res["t0"] = L.lib.orion_now_ns()
    for th in ths:
        th.start()
    prev_mask = os.sched_getaffinity(0) if hp_cpu is not None else None
    try:
        if hp is not None:
            if hp_cpu is not None:
                os.sched_setaffinity(0, {hp_cpu})
            res["hp"] = o.run_requests(hp_id, hp.ops, hp_arrivals, in_cycle=hp.inp.shape[0], out_cycle=hp.n_req)
    except BaseException as e:
        errs.append(e)
    finally:
        if prev_mask is not None:
            os.sched_setaffinity(0, prev_mask)
        for th in ths:          # BE request streams are finite: they end on their own
            th.join()
    res["t1"] = L.lib.orion_now_ns()
    try:
        o.stop()
    except Exception as e:
        errs.append(e)
    if errs:
        o.destroy()
        raise errs[0]
    res["stats"] = o.stats()
    if log_capacity:
        res["log"] = o.read_log()
    o.destroy()
    return res
