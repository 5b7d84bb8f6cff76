// Probe: FP32 FMA throughput per SM of FFMA (3-register) vs packed FFMA2 (fma.rn.f32x2, scalar
// broadcast operand), register-resident, 16 independent accumulators per thread, 8-32 warps per SM.
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void ffma2(float2& d, float a, float2 b) {
  asm volatile("{\n\t.reg .b64 a2, b2, d2;\n\tmov.b64 a2, {%2, %2};\n\tmov.b64 b2, {%3, %4};\n\tmov.b64 d2, {%0, %1};\n\t"
               "fma.rn.f32x2 d2, a2, b2, d2;\n\tmov.b64 {%0, %1}, d2;\n\t}"
               : "+f"(d.x), "+f"(d.y) : "f"(a), "f"(b.x), "f"(b.y));
}

template <bool PACKED>
__global__ void k(int iters, float* out, unsigned long long* cyc) {
  float a = threadIdx.x * 1e-7f, b0 = 1.0001f, b1 = 0.9999f;
  float acc[16];
#pragma unroll
  for (int j = 0; j < 16; j++) acc[j] = j;
  long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
    if (PACKED) {
#pragma unroll
      for (int j = 0; j < 16; j += 2) {
        float2 d = make_float2(acc[j], acc[j + 1]);
        ffma2(d, a, make_float2(b0, b1));
        acc[j] = d.x; acc[j + 1] = d.y;
      }
    } else {
#pragma unroll
      for (int j = 0; j < 16; j++) asm volatile("fma.rn.f32 %0, %1, %2, %0;" : "+f"(acc[j]) : "f"(a), "f"(j & 1 ? b1 : b0));
    }
  }
  long long t1 = clock64();
  float s = 0;
#pragma unroll
  for (int j = 0; j < 16; j++) s += acc[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
  float* o; unsigned long long* c;
  cudaMalloc(&o, 148 * 1024 * 4); cudaMalloc(&c, 148 * 8);
  for (int thr : {256, 512, 1024}) {
    for (int packed = 0; packed < 2; packed++) {
      const int iters = 20000;
      if (packed) k<true><<<148, thr>>>(iters, o, c); else k<false><<<148, thr>>>(iters, o, c);
      cudaDeviceSynchronize();
      unsigned long long h; cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
      printf("%s threads/SM %4d: %.1f FMA/clk/SM\n", packed ? "FFMA2" : "FFMA ", thr, (double)thr * 16 * iters / h);
    }
  }
  return 0;
}
