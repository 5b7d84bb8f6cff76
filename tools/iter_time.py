"""Device time of one client iteration: (a) its ops captured in a CUDA graph (no host gaps),
(b) through liborion's scheduler (dedicated, no throttle). The gap between them is the runtime's
per-op overhead (launch path + completion signal)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import collocate as C

torch.cuda.set_device(0)
for client in sys.argv[1:] or ["be", "hp"]:
    g = bench.build_client("rn50_mnv2", client)
    ops = [(fn, a) for fn, a, lab in g.ops if isinstance(fn, str)]
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for fn, a in ops: orion.kernel_launch(fn, a, s.cuda_stream)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=s):
        for fn, a in ops: orion.kernel_launch(fn, a, s.cuda_stream)
    for _ in range(3): graph.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 10
    e0.record(s)
    for _ in range(n): graph.replay()
    e1.record(s); torch.cuda.synchronize()
    tg = e0.elapsed_time(e1) / n
    if client == "be":
        g.params.reset()
        be = C.BEClient(g)
        C.run_session(be=be, be_iters=3)
        t0 = time.time(); r = C.run_session(be=be, be_iters=20); dt = (time.time() - t0)
        te = r["be_t_end"]
        tsched = (te[-1] - te[0]) / (len(te) - 1) / 1e6
        print(f"{client}: {len(ops)} kernels; CUDA-graph iteration {tg:.3f} ms; via scheduler {tsched:.3f} ms/iteration")
    else:
        print(f"{client}: {len(ops)} kernels; CUDA-graph request {tg:.3f} ms")
