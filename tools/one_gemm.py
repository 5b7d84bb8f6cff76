import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import _lib as L
M, N, K, flags = [int(x) for x in sys.argv[1:5]]
A = torch.randn((K, M) if flags & 1 else (M, K), device="cuda"); B = torch.randn((N, K) if flags & 2 else (K, N), device="cuda")
C = torch.zeros(M, N, device="cuda"); ws = torch.zeros(int(L.lib.orion_gemm_workspace_bytes(M, N, K)) // 4 + 64, device="cuda")
args = [A.data_ptr(), B.data_ptr(), C.data_ptr(), 0, M, N, K, A.shape[1], B.shape[1], N, flags, ws.data_ptr(), ws.numel() * 4]
orion.kernel_launch("gemm", args, torch.cuda.current_stream().cuda_stream); torch.cuda.synchronize()
