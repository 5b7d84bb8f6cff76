"""Conditioning of the full-size ResNet-50 b64 weight-gradient GEMMs (config 3's BE): runs the op
list, then for each flags=1 GEMM reports rel L2 vs the fp64 product, the cancellation ratio
kappa = ||(|A|^T |B|)|| / ||A^T B|| and the worst elementwise error / (4 u sqrt(K) |A|^T |B|)."""
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import torch  # noqa: E402
import paper_conf_eurosys_stratimk24_b200 as orion  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import workloads as W  # noqa: E402
from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info  # noqa: E402
from synth import inputs as si  # noqa: E402
import opcheck  # noqa: E402

torch.cuda.set_device(0)
P = si.make_params(W.resnet_train_spec())
g = W.resnet_train_graph(P, [si.normal((64, 224, 224, 3), si.BE_SEED, sub=0)], [si.labels(64, 1000, si.BE_SEED, sub=0)])
Pm = g.params
tensors = [Pm.flat] + list(g.bufs.values()) + list(Pm.p.values()) + list(Pm.g.values()) + [g._ws]
R = opcheck.Resolver(tensors)
s = torch.cuda.current_stream().cuda_stream
for fn, args, lab in g.ops:
    if isinstance(fn, str):
        orion.kernel_launch(fn, args, s)
torch.cuda.synchronize()
U = 2.0 ** -24
for fn, a, lab in g.ops:
    if fn != "gemm" or a[10] != 1:
        continue
    M, N, K, lda, ldb, ldc = a[4], a[5], a[6], a[7], a[8], a[9]
    A = R.get(a[0], K * lda).view(K, lda)[:, :M].double().cpu()
    B = R.get(a[1], K * ldb).view(K, ldb)[:, :N].double().cpu()
    C = R.get(a[2], M * ldc).view(M, ldc)[:, :N].double().cpu()
    ref = A.t() @ B
    absref = A.abs().t() @ B.abs()
    rel = float((C - ref).norm() / ref.norm())
    kappa = float(absref.norm() / ref.norm())
    worst = float(((C - ref).abs() / (4 * U * math.sqrt(K) * absref + 1e-30)).max())
    kern = kernel_info("gemm", a)["kernel"]
    print(f"{lab:28s} M={M:5d} N={N:5d} K={K:7d} rel={rel:.2e} kappa={kappa:8.1f} rel/kappa={rel / kappa:.2e} "
          f"worst/bound={worst:.3f} {kern[-45:]}", flush=True)
