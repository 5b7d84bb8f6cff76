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
for shp in [(128, 64, 64, 2), (128, 64, 1024, 2), (128, 128, 4096, 2), (256, 128, 1024, 2), (4096, 4096, 4096, 2), (8192, 1024, 2048, 2), (2048, 2048, 8192, 0), (196, 512, 4608, 2), (784, 256, 2304, 2), (3136, 128, 1152, 2),
            (4704, 1280, 320, 2), (1280, 320, 4704, 1), (12544, 64, 576, 2)]:
    run(*shp)
