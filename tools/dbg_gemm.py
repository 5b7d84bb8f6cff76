import sys, torch
sys.path.insert(0, "."); sys.path.insert(0, "tests")
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import _lib as L
from oracle import model as om
from synth import inputs as si
torch.cuda.set_device(0)
def rel(a, b):
    a, b = a.double().cpu(), b.double().cpu(); return float((a - b).norm() / b.norm())
s = torch.cuda.current_stream().cuda_stream
for (M, N, K) in [(3136, 4608, 512), (12544, 2304, 256), (50176, 1152, 128), (200704, 576, 64), (3136, 1280, 512), (3136, 4096, 512), (6272, 4608, 512)]:
    A = si.normal((M, K), 1); B = si.normal((K, N), 2) * 0.05
    C = torch.zeros(M, N, device="cuda")
    ws = torch.zeros(L.lib.orion_gemm_workspace_bytes(M, N, K) // 4 + 64, device="cuda")
    args = [A.cuda().data_ptr(), 0, C.data_ptr(), 0, M, N, K, K, N, N, 0, ws.data_ptr(), ws.numel() * 4]
    Bd = B.cuda(); args[1] = Bd.data_ptr(); Ad = A.cuda(); args[0] = Ad.data_ptr()
    orion.kernel_launch("gemm", args, s); torch.cuda.synchronize()
    grid = orion.runtime.kernel_geometry("gemm", args)
    print(M, N, K, "rel", rel(C, A.double() @ B.double()), "geom", grid, flush=True)
