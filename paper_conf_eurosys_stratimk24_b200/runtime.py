"""Thin Python face of liborion (same names as include/orion.h; marshalling only)."""
import ctypes
import struct

import numpy as np

from . import _lib as L
from ._lib import Op, Config, check


def f32bits(x):
    return struct.unpack("<I", struct.pack("<f", float(x)))[0]


def make_op(fn, args, kernel_id=0, cls=L.CLS_U, sm_needed=0, dur_ns=0, kind=L.OP_KERNEL, opflags=0):
    """Build an orion_op record (orion.h). args: ints (device pointers from tensor.data_ptr(), dims,
    fp32 bit patterns)."""
    op = Op()
    op.fn = L.FN[fn] if isinstance(fn, str) else int(fn)
    op.kind = kind
    op.nargs = len(args)
    op.opflags = opflags
    op.prof.kernel_id = kernel_id
    op.prof.cls = cls
    op.prof.sm_needed = sm_needed
    op.prof.dur_ns = dur_ns
    for i, a in enumerate(args):
        op.args[i] = int(a) & 0xFFFFFFFFFFFFFFFF
    return op


def op_array(ops):
    arr = (Op * len(ops))()
    for i, o in enumerate(ops):
        arr[i] = o
    return arr


class Orion:
    """One instance per GPU."""

    def __init__(self, device=0, backend=L.BACKEND_CUDA, num_sms=0, sm_threshold=0, dur_threshold_ppm=25000,
                 hp_latency_ns=0, be_partition_sms=0, flags=0, queue_capacity=4096, sched_cpu=-1, log_capacity=0,
                 fake_time_scale_pct=100, trace_kernel_id=None, fake_contention=False):
        cfg = Config()
        cfg.num_sms, cfg.sm_threshold, cfg.dur_threshold_ppm = num_sms, sm_threshold, dur_threshold_ppm
        cfg.be_partition_sms, cfg.hp_latency_ns, cfg.flags = be_partition_sms, hp_latency_ns, flags
        cfg.queue_capacity, cfg.backend, cfg.sched_cpu = queue_capacity, backend, sched_cpu
        cfg.log_capacity, cfg.fake_time_scale_pct = log_capacity, fake_time_scale_pct
        cfg.fake_contention = 1 if fake_contention else 0
        cfg.trace_kernel_id_plus1 = 0 if trace_kernel_id is None else trace_kernel_id + 1
        self.h = ctypes.c_void_p()
        check(L.lib.orion_create(device, ctypes.byref(cfg), ctypes.byref(self.h)), "orion_create")
        self.started = False

    def register_client(self, prio):
        cid = ctypes.c_int()
        check(L.lib.orion_register_client(self.h, prio, ctypes.byref(cid)), "orion_register_client")
        return cid.value

    def client_stream(self, cid):
        s = ctypes.c_void_p()
        check(L.lib.orion_client_stream(self.h, cid, ctypes.byref(s)), "orion_client_stream")
        return s.value

    def start(self):
        check(L.lib.orion_start(self.h), "orion_start")
        self.started = True

    def submit(self, cid, op):
        seq = ctypes.c_uint64()
        rc = L.lib.orion_submit(self.h, cid, ctypes.byref(op), ctypes.byref(seq))
        if rc == L.E_AGAIN:
            return None
        check(rc, "orion_submit")
        return seq.value

    def submit_n(self, cid, arr):
        first = ctypes.c_uint64()
        rc = L.lib.orion_submit_n(self.h, cid, arr, len(arr), ctypes.byref(first))
        if rc == L.E_AGAIN:
            return None
        check(rc, "orion_submit_n")
        return first.value

    def synchronize(self, cid, timeout_ns=0):
        check(L.lib.orion_synchronize(self.h, cid, timeout_ns), "orion_synchronize")

    def done_seq(self, cid):
        d = ctypes.c_uint64()
        check(L.lib.orion_done_seq(self.h, cid, ctypes.byref(d)), "orion_done_seq")
        return d.value

    def stop(self):
        check(L.lib.orion_stop(self.h), "orion_stop")
        self.started = False

    def read_log(self):
        need = ctypes.c_size_t()
        rc = L.lib.orion_read_log(self.h, None, 0, ctypes.byref(need))
        if rc not in (L.OK, L.E_NOMEM):
            check(rc, "orion_read_log")
        buf = ctypes.create_string_buffer(need.value)
        check(L.lib.orion_read_log(self.h, buf, need.value, ctypes.byref(need)), "orion_read_log")
        return buf.raw[:need.value]

    def trace_read(self):
        """Live durations (ms) of the traced kernel's launches (config trace_kernel_id)."""
        n = ctypes.c_uint32()
        check(L.lib.orion_trace_read(self.h, None, 0, ctypes.byref(n)), "orion_trace_read")
        buf = (ctypes.c_float * max(n.value, 1))()
        check(L.lib.orion_trace_read(self.h, buf, n.value, ctypes.byref(n)), "orion_trace_read")
        return [buf[i] for i in range(n.value)]

    def stats(self):
        out = (ctypes.c_uint64 * 8)()
        check(L.lib.orion_stats(self.h, out, 8), "orion_stats")
        keys = ["iterations", "hp_launches", "be_admits", "be_defers", "memops", "resets", "launch_errors", "launch_ns"]
        return dict(zip(keys, list(out)))

    def run_requests(self, cid, ops, arrivals_ns, in_cycle=1, out_cycle=1):
        """Native open-loop request driver (orion_run_requests). Returns (t_arrival, t_done) ns arrays."""
        arr = op_array(ops)
        arrivals = np.ascontiguousarray(arrivals_ns, dtype=np.int64)
        n = len(arrivals)
        ta = np.zeros(n, dtype=np.int64)
        td = np.zeros(n, dtype=np.int64)
        check(L.lib.orion_run_requests(self.h, cid, arr, len(ops), arrivals.ctypes.data, n, in_cycle, out_cycle,
                                       ta.ctypes.data, td.ctypes.data), "orion_run_requests")
        return ta, td

    def run_requests_direct(self, cid, ops, arrivals_ns, in_cycle=1, out_cycle=1):
        """The native arm (orion_run_requests_direct: direct launches, no scheduler; instance never started)."""
        arr = op_array(ops)
        arrivals = np.ascontiguousarray(arrivals_ns, dtype=np.int64)
        n = len(arrivals)
        ta = np.zeros(n, dtype=np.int64)
        td = np.zeros(n, dtype=np.int64)
        check(L.lib.orion_run_requests_direct(self.h, cid, arr, len(ops), arrivals.ctypes.data, n, in_cycle, out_cycle,
                                              ta.ctypes.data, td.ctypes.data), "orion_run_requests_direct")
        return ta, td

    def run_iterations(self, cid, variants, stop_flag=None, max_iters=0, cap=1 << 16):
        """Native closed-loop training driver (orion_run_iterations). variants: list of op lists."""
        n_ops = len(variants[0])
        flat = op_array([o for v in variants for o in v])
        t_end = np.zeros(cap, dtype=np.int64)
        iters = ctypes.c_uint64()
        stop_ptr = ctypes.addressof(stop_flag) if stop_flag is not None else None
        check(L.lib.orion_run_iterations(self.h, cid, flat, n_ops, len(variants), stop_ptr, max_iters,
                                         t_end.ctypes.data, cap, ctypes.byref(iters)), "orion_run_iterations")
        return t_end[:iters.value]

    def destroy(self):
        if self.h:
            L.lib.orion_destroy(self.h)
            self.h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def now_ns():
    return L.lib.orion_now_ns()


def kernel_launch(fn, args, stream=0):
    """Direct launch of one operator (no scheduler): the profiler's solo runner and op-level tests."""
    a = (ctypes.c_uint64 * len(args))(*[int(x) & 0xFFFFFFFFFFFFFFFF for x in args])
    check(L.lib.orion_kernel_launch(L.FN[fn] if isinstance(fn, str) else fn, a, len(args), ctypes.c_void_p(stream)),
          f"kernel_launch({fn})")


def kernel_geometry(fn, args):
    a = (ctypes.c_uint64 * len(args))(*[int(x) & 0xFFFFFFFFFFFFFFFF for x in args])
    grid = ctypes.c_uint64()
    bps, thr, smem = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    check(L.lib.orion_kernel_geometry(L.FN[fn] if isinstance(fn, str) else fn, a, len(args), ctypes.byref(grid),
                                      ctypes.byref(bps), ctypes.byref(thr), ctypes.byref(smem)), f"kernel_geometry({fn})")
    return grid.value, bps.value, thr.value, smem.value


def kernel_info(fn, args):
    """orion_kernel_info: launch geometry, registers, shared memory, occupancy and pipe of one op as it
    would launch (the offline profiler's inputs)."""
    a = (ctypes.c_uint64 * len(args))(*[int(x) & 0xFFFFFFFFFFFFFFFF for x in args])
    info = L.KernelInfo()
    check(L.lib.orion_kernel_info(L.FN[fn] if isinstance(fn, str) else fn, a, len(args), ctypes.byref(info)),
          f"kernel_info({fn})")
    d = {k: getattr(info, k) for k, _ in info._fields_}
    d["kernel"] = d["kernel"].decode(errors="replace")
    return d
