// Probe: tcgen05.mma issue rate on one SM (kind::tf32 and kind::f16, M = 128, SWIZZLE_NONE
// K-major smem operands), back-to-back into one accumulator vs rotating accumulators; and the
// throughput of cvt.rna.tf32.f32. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma_rate mma_rate.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}

template <int KIND>   // 0 tf32, 1 f16(bf16)
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  if (KIND == 0)
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
  else
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}

// MN-major tf32 operand descriptor: 128-byte swizzle with 32-byte atoms (layout type 1), LBO 4 KB
// between MN atoms, SBO 512 B between 4-row k-groups (the weight-gradient kernels' layout)
__device__ __forceinline__ uint64_t desc_mn(uint32_t addr) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)(4096 >> 4) << 16) | ((uint64_t)(512 >> 4) << 32) | (1ull << 46) | (1ull << 61);
}

template <int KIND, int N, int NACC, bool MN = false>
__global__ void __launch_bounds__(128, 1) k_mma(int iters, unsigned long long* out) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint32_t slot;
  __shared__ __align__(8) uint64_t bar;
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0;
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&slot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = slot;
  if (threadIdx.x == 0) {
    constexpr uint32_t ab = KIND == 0 ? 2u : 1u;
    const uint32_t mn = MN ? ((1u << 15) | (1u << 16)) : 0u;
    const uint32_t idesc = (1u << 4) | (ab << 7) | (ab << 10) | mn | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    const uint32_t base = (smem_u32(sm) + 1023u) & ~1023u;
    const uint64_t da = MN ? desc_mn(base) : sdesc(base, 128, 256), db = MN ? desc_mn(base + 32768) : sdesc(base + 32768, 128, 256);
    long long t0 = clock64();
    for (int i = 0; i < iters; i++) {
#pragma unroll
      for (int j = 0; j < 6; j++) {
        const int a = (i * 6 + j) % NACC;
        mma<KIND>(tmem + (uint32_t)(a * N), da, db, idesc, (i | j) != 0);
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
    uint32_t ok = 0;
    while (!ok) {
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
    }
    long long t1 = clock64();
    out[blockIdx.x] = (unsigned long long)(t1 - t0);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
  }
}

__global__ void k_cvt(int iters, float* out, unsigned long long* cyc) {
  float x = threadIdx.x * 1.1f, acc = 0.f;
  long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
    uint32_t u;
    asm volatile("cvt.rna.tf32.f32 %0, %1;" : "=r"(u) : "f"(x));
    acc += __uint_as_float(u);
    x += 1.0f;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = (unsigned long long)(t1 - t0);
}

template <int KIND, int N, int NACC, bool MN = false>
void run(const char* name) {
  unsigned long long* d;
  cudaMalloc(&d, 148 * 8);
  auto f = k_mma<KIND, N, NACC, MN>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  const int iters = 2000;
  f<<<148, 128, 65536>>>(iters, d);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  double cyc = (double)h[0] / (iters * 6);
  const int K = KIND == 0 ? 8 : 16;
  printf("%-34s %s  cycles/MMA %.1f  FMA/clk/SM %.0f\n", name, cudaGetErrorString(e), cyc, 128.0 * N * K / cyc);
  cudaFree(d);
}

int main() {
  run<0, 32, 1>("tf32 N=32  same acc");
  run<0, 32, 4>("tf32 N=32  4 accs");
  run<0, 32, 1, true>("tf32 MN-major N=32 same acc");
  run<0, 32, 4, true>("tf32 MN-major N=32 4 accs");
  run<0, 64, 4, true>("tf32 MN-major N=64 4 accs");
  run<0, 128, 3, true>("tf32 MN-major N=128 3 accs");
  run<0, 64, 1>("tf32 N=64  same acc");
  run<0, 64, 4>("tf32 N=64  4 accs");
  run<0, 128, 1>("tf32 N=128 same acc");
  run<0, 128, 3>("tf32 N=128 3 accs");
  run<0, 256, 1>("tf32 N=256 same acc");
  run<0, 256, 2>("tf32 N=256 2 accs");
  run<1, 128, 1>("bf16 N=128 same acc");
  run<1, 256, 1>("bf16 N=256 same acc");
  run<1, 256, 2>("bf16 N=256 2 accs");
  float* o; unsigned long long* c;
  cudaMalloc(&o, 148 * 256 * 4); cudaMalloc(&c, 148 * 8);
  k_cvt<<<148, 256>>>(10000, o, c);
  cudaDeviceSynchronize();
  unsigned long long h; cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
  printf("cvt.rna.tf32 (+fadd) 256 thr/SM: %.2f cycles per iteration per thread -> %.1f cvt/clk/SM\n", (double)h / 10000, 256.0 * 10000 / h);
  return 0;
}
