"""Where an HP request's latency goes: host launch cost vs device time of its kernel ops.

  host   : wall time of issuing every kernel op of the client once (no sync), per launch
  direct : wall time of issue + completion (sync) = the direct-launch request latency w/o copies
  device : one CUDA-graph replay of the same launches (device time, launch gaps ~ graph's)
Usage: python tools/diag_launch.py [config] [client]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import _lib as L  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "rn50_mnv2"
    client = sys.argv[2] if len(sys.argv) > 2 else "hp"
    torch.cuda.set_device(0)
    g = bench.build_client(cfg, client)
    ops = [(L.FN[fn], (__import__("ctypes").c_uint64 * len(args))(*[int(x) & 0xFFFFFFFFFFFFFFFF for x in args]), len(args))
           for fn, args, _ in g.ops if isinstance(fn, str)]
    st = torch.cuda.Stream()
    s = st.cuda_stream
    lib = L.lib

    def issue():
        for fn, a, n in ops:
            lib.orion_kernel_launch(fn, a, n, s)

    for _ in range(3):
        issue()
    torch.cuda.synchronize()
    host, direct = [], []
    for _ in range(20):
        t0 = time.perf_counter()
        issue()
        t1 = time.perf_counter()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        host.append(t1 - t0)
        direct.append(t2 - t0)
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr, stream=st):
        issue()
    gr.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    dev = []
    for _ in range(10):
        e0.record()
        gr.replay()
        e1.record()
        torch.cuda.synchronize()
        dev.append(e0.elapsed_time(e1) / 1e3)
    orion_p50 = None
    if client == "hp":   # the native request path (H2D input, kernels with completion signals, D2H logits)
        import numpy as np
        from paper_conf_eurosys_stratimk24_b200 import collocate as C
        hp = C.HPClient(g, bench.hp_inputs(cfg, 8) if hasattr(bench, "hp_inputs") else [torch.zeros(g.x.numel())], 200)
        spaced = (np.arange(1, 101) * 10e6).astype(np.int64)
        C.run_direct(hp, spaced[:10])
        rn = C.run_direct(hp, spaced)
        orion_p50 = float(np.median(rn["t_done"] - rn["t_arrival"])) / 1e6
    med = lambda v: sorted(v)[len(v) // 2]  # noqa: E731
    n = len(ops)
    print(f"{cfg}/{client}: {n} kernel ops")
    print(f"  host issue      {med(host) * 1e3:8.3f} ms  ({med(host) / n * 1e6:5.2f} us per launch, ctypes + geom + launch)")
    print(f"  direct (sync)   {med(direct) * 1e3:8.3f} ms")
    print(f"  graph replay    {med(dev) * 1e3:8.3f} ms  ({med(dev) / n * 1e6:5.2f} us per kernel incl. graph launch gaps)")
    if orion_p50 is not None:
        print(f"  native request  {orion_p50:8.3f} ms  (orion_run_requests_direct p50: + H2D / D2H, completion signals)")


if __name__ == "__main__":
    main()
