"""Microbenchmark of liborion's reduction operators (BN stats / backward reduce, depthwise wgrad) at
MobileNetV2 b96 shapes: CUDA-event time per launch (solo, warm), achieved GB/s of compulsory bytes."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import _lib as L


def timeit(fn, args, reps=20):
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):
        orion.kernel_launch(fn, args, s)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        orion.kernel_launch(fn, args, s)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3   # us


def ws(nbytes):
    return torch.zeros(int(nbytes) // 4 + 64, device="cuda")


def bn(rows, C):
    x = torch.randn(rows, C, device="cuda")
    dy = torch.randn(rows, C, device="cuda")
    v = [torch.zeros(C, device="cuda") for _ in range(6)]
    w = ws(L.lib.orion_bn_workspace_bytes(rows, C))
    a = [x.data_ptr(), v[0].data_ptr(), v[1].data_ptr(), v[2].data_ptr(), v[3].data_ptr(), rows, C, orion.f32bits(1e-5),
         orion.f32bits(0.1), w.data_ptr(), w.numel() * 4]
    t = timeit("bn_stats", a)
    g = orion.kernel_geometry("bn_stats", a)[0]
    b = [x.data_ptr(), dy.data_ptr(), v[0].data_ptr(), v[1].data_ptr(), v[4].data_ptr(), v[5].data_ptr(), rows, C, w.data_ptr(),
         w.numel() * 4]
    t2 = timeit("bn_bwd_reduce", b)
    print(f"bn rows={rows:8d} C={C:5d} grid={g:5d}  stats {t:7.1f} us {rows*C*4/t/1e3:6.0f} GB/s   bwd_reduce {t2:7.1f} us "
          f"{rows*C*8/t2/1e3:6.0f} GB/s")


def dw(n, h, c, stride):
    p = (h - 1) // stride + 1
    x = torch.randn(n, h, h, c, device="cuda")
    dy = torch.randn(n, p, p, c, device="cuda")
    dwt = torch.zeros(c, 9, device="cuda")
    w = ws(L.lib.orion_dw_wgrad_workspace_bytes(n, c, p, p))
    a = [x.data_ptr(), dy.data_ptr(), dwt.data_ptr(), n, h, h, c, c, 3, 3, stride, 1, p, p, w.data_ptr(), w.numel() * 4]
    t = timeit("dw_wgrad", a)
    g = orion.kernel_geometry("dw_wgrad", a)[0]
    byt = (x.numel() + dy.numel()) * 4
    print(f"dw_wgrad n={n} h={h:4d} c={c:5d} s={stride} grid={g:5d}  {t:7.1f} us {byt/t/1e3:6.0f} GB/s")


if __name__ == "__main__":
    torch.cuda.set_device(0)
    if len(sys.argv) > 1:   # one case: bn ROWS C | dw N H C STRIDE
        {"bn": bn, "dw": dw}[sys.argv[1]](*[int(v) for v in sys.argv[2:]])
        sys.exit(0)
    for rows, C in [(1204224, 32), (1204224, 96), (301056, 96), (301056, 144), (301056, 24), (75264, 192), (75264, 32),
                    (18816, 64), (18816, 384), (4704, 160), (4704, 960), (4704, 1280)]:
        bn(rows, C)
    for n, h, c, s in [(96, 112, 32, 1), (96, 112, 96, 2), (96, 56, 144, 1), (96, 56, 144, 2), (96, 28, 192, 1), (96, 14, 384, 1),
                       (96, 7, 960, 1)]:
        dw(n, h, c, s)
