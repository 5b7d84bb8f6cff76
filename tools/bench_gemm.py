"""Microbenchmark of liborion's GEMM paths (event-timed, solo)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import _lib as L

def run(M, N, K, flags, reps=10):
    A = torch.randn((K, M) if flags & 1 else (M, K), device="cuda")
    B = torch.randn((N, K) if flags & 2 else (K, N), device="cuda")
    C = torch.zeros(M, N, device="cuda")
    wsb = int(L.lib.orion_gemm_workspace_bytes(M, N, K))
    ws = torch.zeros(max(wsb // 4, 1) + 64, device="cuda")
    args = [A.data_ptr(), B.data_ptr(), C.data_ptr(), 0, M, N, K, A.shape[1], B.shape[1], N, flags, ws.data_ptr(), ws.numel() * 4]
    s = torch.cuda.current_stream().cuda_stream
    grid, bps, thr, smem = orion.kernel_geometry("gemm", args)
    for _ in range(3): orion.kernel_launch("gemm", args, s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(reps): orion.kernel_launch("gemm", args, s)
    e1.record(); torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / reps * 1e-3
    print(f"M={M:6d} N={N:5d} K={K:6d} fl={flags} grid={grid:5d} thr={thr} smem={smem:6d}  {t*1e6:9.1f} us  {2*M*N*K/t/1e12:7.2f} TF/s")

torch.cuda.set_device(0)
SHAPES = {
    "generic": [(4096, 4096, 4096, 2), (8192, 1024, 2048, 2), (196, 512, 4608, 2), (784, 256, 2304, 2), (3136, 128, 1152, 2),
                (4704, 1280, 320, 2), (1280, 320, 4704, 1), (12544, 64, 576, 2)],
    # MobileNetV2 b96 1x1 convs: fwd (flags 2: x [M][Cin] . W[Cout][Cin]^T) and dgrad (flags 0: dy [M][Cout] . W[Cout][Cin])
    "dbg": [(1204224, 96, 16, 2), (301056, 24, 144, 2), (1204224, 16, 96, 0), (4704, 1280, 320, 2)],
    "mnv2": [(1204224, 16, 32, 2), (1204224, 96, 16, 2), (301056, 24, 96, 2), (301056, 144, 24, 2), (301056, 24, 144, 2),
             (75264, 32, 144, 2), (75264, 192, 32, 2), (75264, 32, 192, 2), (18816, 384, 64, 2), (18816, 64, 384, 2),
             (18816, 576, 96, 2), (4704, 960, 160, 2), (4704, 160, 960, 2), (4704, 1280, 320, 2),
             (1204224, 32, 16, 0), (1204224, 16, 96, 0), (301056, 96, 24, 0), (301056, 24, 144, 0), (75264, 144, 32, 0),
             (75264, 32, 192, 0), (18816, 64, 384, 0), (4704, 160, 960, 0), (4704, 320, 1280, 0)],
}
for name in (sys.argv[1:] or ["generic", "mnv2"]):
    for shp in SHAPES[name]:
        run(*shp)
