#!/bin/bash
mkdir -p gpurun_out
# probe binaries are build outputs (git-ignored): compile them here
for b in probe mma_rate tma_tf32; do nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o tools/probe/$b tools/probe/$b.cu -lcuda || exit 1; done
{ nproc; lscpu | head -20; nvidia-smi; nvidia-smi topo -m; free -g; } > gpurun_out/box_info.txt 2>&1
./tools/probe/probe > gpurun_out/probe.txt 2>&1
python - >> gpurun_out/probe.txt 2>&1 <<'PY'
import torch,time
torch.backends.cuda.matmul.allow_tf32=True
a=torch.randn(8192,8192,device='cuda'); b=torch.randn(8192,8192,device='cuda')
for _ in range(3): c=a@b
torch.cuda.synchronize(); best=1e9
for _ in range(10):
  s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True); s.record(); c=a@b; e.record(); torch.cuda.synchronize(); best=min(best,s.elapsed_time(e))
print("tf32 8192^3 TFLOPS", 2*8192**3/best/1e9)
torch.backends.cuda.matmul.allow_tf32=False
for _ in range(2): c=a@b
torch.cuda.synchronize(); best=1e9
for _ in range(5):
  s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True); s.record(); c=a@b; e.record(); torch.cuda.synchronize(); best=min(best,s.elapsed_time(e))
print("fp32 (no tf32) 8192^3 TFLOPS", 2*8192**3/best/1e9)
PY
