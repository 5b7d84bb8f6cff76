// Probe: (1) does kind::tf32 truncate or round the low 13 mantissa bits of fp32 smem operands?
// (2) does a 3-D tensor map {4 floats, rows, K/4} with strides {ld*4, 16 B} load a K-major
// SWIZZLE_NONE core-matrix tile (q * rows * 16 + r * 16 + e * 4) in one TMA op?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_tf32 tma_tf32.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cmath>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}

// D[m][n] = sum_k A[m][k] B[n][k], M = 128, N = 16, K = 8, K-major no swizzle (core matrices 8 rows x 16 B;
// LBO = 128 B between the two k-halves, SBO = 256 B between 8-row groups)
__global__ void k_trunc(const float* A, const float* B, float* D) {
  __shared__ __align__(1024) float sa[128 * 8];
  __shared__ __align__(1024) float sb[16 * 8];
  __shared__ uint32_t slot;
  __shared__ __align__(8) uint64_t bar;
  const int t = threadIdx.x;
  for (int k = 0; k < 8; k++) {   // element (row, k): half = k / 4, e = k % 4
    const int off = (t >> 3) * 64 + (k >> 2) * 32 + (t & 7) * 4 + (k & 3);
    sa[off] = A[t * 8 + k];
    if (t < 16) sb[off] = B[t * 8 + k];
  }
  if (t < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(smem_u32(&slot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (t == 0) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)) : "memory"); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = slot;
  if (t == 0) {
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(16 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                 "l"(sdesc(smem_u32(sa), 128, 256)), "l"(sdesc(smem_u32(sb), 128, 256)), "r"(idesc), "r"(0u) : "memory");
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
  }
  uint32_t ok = 0;
  while (!ok) asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  uint32_t r[16];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]),
                 "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
               : "r"(tmem + ((uint32_t)((t / 32) * 32) << 16)));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  for (int n = 0; n < 16; n++) D[t * 16 + n] = __uint_as_float(r[n]);
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tmem) : "memory");
}

__global__ void k_tma(const __grid_constant__ CUtensorMap tm, float* out, int k0, int m0) {
  __shared__ __align__(1024) float s[4 * 128 * 4];
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar)), "r"(8192) : "memory");
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(smem_u32(s)),
                 "l"(&tm), "r"(0), "r"(m0), "r"(k0 / 4), "r"(smem_u32(&bar)) : "memory");
    uint32_t ok = 0;
    while (!ok) asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(smem_u32(&bar)) : "memory");
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) out[i] = s[i];
}

int main() {
  // (1) truncation vs rounding
  float hA[128 * 8], hB[16 * 8], hD[128 * 16];
  for (int m = 0; m < 128; m++)
    for (int k = 0; k < 8; k++) {
      uint32_t u = 0x3F800000u | ((uint32_t)(m * 37 + 5) & 0x1FFFu) | ((uint32_t)m << 13 & 0x7FE000u);   // low 13 bits set
      float f; memcpy(&f, &u, 4); hA[m * 8 + k] = k == 0 ? f : 0.f;
    }
  for (int n = 0; n < 16; n++)
    for (int k = 0; k < 8; k++) hB[n * 8 + k] = (n == 0 && k == 0) ? 1.f : 0.f;
  float *dA, *dB, *dD;
  cudaMalloc(&dA, sizeof(hA)); cudaMalloc(&dB, sizeof(hB)); cudaMalloc(&dD, sizeof(hD));
  cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice); cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
  k_trunc<<<1, 128>>>(dA, dB, dD);
  printf("k_trunc: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
  int n_tr = 0, n_rn = 0, n_other = 0;
  for (int m = 0; m < 128; m++) {
    uint32_t u; memcpy(&u, &hA[m * 8], 4);
    uint32_t tr = u & 0xFFFFE000u;
    uint32_t rn = (u + 0x1000u) & 0xFFFFE000u;
    uint32_t d; memcpy(&d, &hD[m * 16], 4);
    if (d == tr) n_tr++; else if (d == rn) n_rn++; else n_other++;
    if (m < 4) printf("  x=%08x trunc=%08x rn=%08x mma=%08x\n", u, tr, rn, d);
  }
  printf("tf32 operand: truncated %d, rounded %d, other %d (of 128)\n", n_tr, n_rn, n_other);

  // (2) 3-D tensor map K-major core-matrix tile
  const int M = 300, K = 40;
  float* hX = new float[M * K];
  for (int i = 0; i < M * K; i++) hX[i] = (float)i;
  float *dX, *dO; cudaMalloc(&dX, M * K * 4); cudaMalloc(&dO, 2048 * 4);
  cudaMemcpy(dX, hX, M * K * 4, cudaMemcpyHostToDevice);
  CUtensorMap tm;
  cuuint64_t dims[3] = {4, (cuuint64_t)M, (cuuint64_t)(K / 4)};
  cuuint64_t strides[2] = {(cuuint64_t)K * 4, 16};
  cuuint32_t box[3] = {4, 128, 4};
  cuuint32_t es[3] = {1, 1, 1};
  CUresult r = cuTensorMapEncodeTiled(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, dX, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode 3d: %d\n", (int)r);
  if (r == CUDA_SUCCESS) {
    const int m0 = 256, k0 = 32;   // ragged: rows 256..299 valid (44), k 32..39 valid (2 chunks)
    k_tma<<<1, 128>>>(tm, dO, k0, m0);
    printf("k_tma: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    float hO[2048]; cudaMemcpy(hO, dO, sizeof(hO), cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int q = 0; q < 4; q++)
      for (int rr = 0; rr < 128; rr++)
        for (int e = 0; e < 4; e++) {
          const int m = m0 + rr, k = k0 + 4 * q + e;
          const float want = (m < M && k < K) ? hX[m * K + k] : 0.f;
          if (hO[q * 512 + rr * 4 + e] != want) { if (bad < 5) printf("  mismatch q%d r%d e%d got %f want %f\n", q, rr, e, hO[q * 512 + rr * 4 + e], want); bad++; }
        }
    printf("3d TMA core-matrix tile: %d mismatches of 2048\n", bad);
  }
  return 0;
}
