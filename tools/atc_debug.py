"""Bring-up check of atc.cu's TMA / UMMA layouts (ORION_ATC_DBG=1: the stage-0 A tile decoded from
shared memory through the SW128 MN-major atom formula must equal A^T)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import _lib as L  # noqa: E402
from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info  # noqa: E402

torch.cuda.set_device(0)
M, N, K = 128, 64, 128
A = torch.randn(K, M, device="cuda")
B = torch.randn(K, N, device="cuda")
C = torch.zeros(M, N, device="cuda")
w = torch.zeros(int(L.lib.orion_gemm_workspace_bytes(M, N, K)) // 4 + 64, device="cuda")
a = [A.data_ptr(), B.data_ptr(), C.data_ptr(), 0, M, N, K, M, N, N, 1, w.data_ptr(), w.numel() * 4]
print(kernel_info("gemm", a))
orion.kernel_launch("gemm", a, torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
dbg = os.environ.get("ORION_ATC_DBG", "0")
if dbg == "1":
    ref = A[:32, :].t()   # C[m][k] = A[k][m], k < 32
    got = C[:, :32]
    print("layout decode max err", float((got - ref).abs().max()), "nonzero", int((got != 0).sum()))
    print(got[:3, :6], ref[:3, :6])
else:
    ref = A.double().t() @ B.double()
    print("rel", float((C.double() - ref).norm() / ref.norm()), "nonzero", int((C != 0).sum()))
    print(C[:2, :6], ref[:2, :6])
