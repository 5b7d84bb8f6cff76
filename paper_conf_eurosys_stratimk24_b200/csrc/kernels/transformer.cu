// bf16 transformer operators (HP of BASELINE config 3: BERT-base inference, batch 8, seq 128,
// model cast to bfloat16 and run by PyTorch eager) and the max-pool backward of the
// ResNet training client (BE of config 3).
//
//  * gemm_bf16: y = x W^T + b on the 5th-gen tensor cores (tcgen05.mma kind::f16, bf16 operands,
//    fp32 accumulator in TMEM), operands brought in by TMA (128-byte swizzle) through a 6-8 stage
//    mbarrier ring, one elected MMA thread; epilogue TMEM -> registers -> bias -> bf16 (RNE).
//  * attention: fused scaled-dot-product attention (the one SDPA kernel PyTorch dispatches),
//    per (batch, head, 64-query block); Q K^T and P V on mma.sync m16n8k16 bf16 with fp32
//    accumulators, softmax in fp32 registers, P rounded to bf16 for the second product (what a
//    flash-style kernel does), O normalised and rounded once.
//  * layernorm (warp per row, two-pass mean / variance in registers), gelu (erf), add, embedding
//    gather-sum: 128-bit vectorised (8 bf16 per access), fp32 arithmetic, one rounding per output.
//  * maxpool_bwd (fp32): gather form — each input element sums the gradients of the (at most 4)
//    windows whose first maximum it is, in fixed order; no atomics, so deterministic.
// Every kernel computes each output in one thread (or one warp) in a fixed order: outputs are
// bitwise identical solo and collocated.
#include <cuda.h>
#include <cuda_bf16.h>
#include <float.h>
#include <atomic>

#include "common.cuh"

namespace {

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

typedef __nv_bfloat16 bf16;

__device__ __forceinline__ float bf2f(bf16 v) { return __bfloat162float(v); }
__device__ __forceinline__ uint32_t pack_bf2(float lo, float hi) {
  __nv_bfloat162 t = __floats2bfloat162_rn(lo, hi);   // .x = lo (low 16 bits), .y = hi
  return *reinterpret_cast<uint32_t*>(&t);
}
__device__ __forceinline__ void unpack8(const uint4& u, float* f) {
  const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; i++) { float2 t = __bfloat1622float2(h[i]); f[2 * i] = t.x; f[2 * i + 1] = t.y; }
}
__device__ __forceinline__ uint4 pack8(const float* f) {
  uint4 u;
  u.x = pack_bf2(f[0], f[1]); u.y = pack_bf2(f[2], f[3]); u.z = pack_bf2(f[4], f[5]); u.w = pack_bf2(f[6], f[7]);
  return u;
}

// =============================================================================== gemm_bf16
// TMA-fed tcgen05 GEMM: one thread issues two 2-D tensor copies per stage (A: 128 x 64 bf16, W:
// BN x 64 bf16, 128-byte swizzle, zero fill out of bounds) onto an mbarrier with an expected byte
// count; one thread issues 4 tcgen05.mma (K = 16 each) per stage from the swizzled tiles and
// commits the stage back to the producer; four epilogue warps read the fp32 accumulator from
// TMEM, add the bias (staged in shared memory once), round to bf16 and store through a padded
// shared tile with coalesced 16-byte row stores. One output tile per CTA, fixed k order.
namespace tcb {

constexpr int BM = 128, BK = 64, NTHR = 192;   // warps 0-3 epilogue, 4 TMA producer, 5 MMA issuer / TMEM owner
constexpr int TMA_WARP = 4, MMA_WARP = 5;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t a, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(a), "r"(parity) : "memory");
  }
}
__device__ __forceinline__ void tma2d(uint32_t dst, const CUtensorMap* tm, int c0, int c1, uint32_t bar) {
  asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst), "l"(tm),
               "r"(c0), "r"(c1), "r"(bar) : "memory");
}
// UMMA descriptor, K-major SWIZZLE_128B: 8-row atoms of 128-byte rows (64 bf16), SBO = 1024 B between
// atoms, LBO unused (1), version 1 (bit 46), layout type 2 (bits 61-63); K step j (16 bf16 = 32 B)
// advances the start address by 32 B inside the swizzle atom.
__device__ __forceinline__ uint64_t sdesc128(uint32_t addr) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | (1ull << 16) | ((uint64_t)(1024 >> 4) << 32) | (1ull << 46) | (2ull << 61);
}
__device__ __forceinline__ void mma_bf16(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
               ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t mbar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(mbar) : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float* v) {
  uint32_t r[32];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 32; i++) v[i] = __uint_as_float(r[i]);
}

template <int BN>
struct Cfg {
  static constexpr int A_BYTES = BM * BK * 2, B_BYTES = BN * BK * 2, STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (192 * 1024) / STAGE_BYTES;   // 4 (BN 256) / 6 (BN 128) / 8 (BN 64)
  static constexpr int EPI_LD = BN + 8;                        // padded bf16 staging row
  static constexpr int EPI_BYTES = BM * EPI_LD * 2;
  static constexpr int MAIN = STAGES * STAGE_BYTES > EPI_BYTES ? STAGES * STAGE_BYTES : EPI_BYTES;
  static constexpr int SMEM = MAIN + BN * 4 + 256 + 1024;
  static constexpr int TMEM_COLS = BN;
  static constexpr uint32_t TX = STAGE_BYTES;
  // instruction descriptor (kind::f16): D f32 (bits 4-5 = 1), A bf16 (bits 7-9 = 1), B bf16 (bits
  // 10-12 = 1), both K-major, N >> 3 at bits 17-22, M >> 4 at bits 24-28
  static constexpr uint32_t IDESC = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
};

template <int BN>
__global__ void __launch_bounds__(NTHR, 1) gemm_bf16_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW,
                                                           bf16* __restrict__ C, const bf16* __restrict__ bias, int M, int N, int K,
                                                           OrionSig sig) {
  using Cf = Cfg<BN>;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  // offset the shared array itself (not a uintptr_t round trip), so accesses stay LDS/STS
  unsigned char* smem = smem_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_raw) & 1023u)) & 1023u);
  constexpr int S = Cf::STAGES;
  float* bias_s = reinterpret_cast<float*>(smem + Cf::MAIN);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + Cf::MAIN + BN * 4);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * S + 1);
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + S), done_bar = smem_u32(bars + 2 * S);
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  const int nk = (K + BK - 1) / BK;

  if (tid == 0) {
    for (int s = 0; s < S; s++) { mbar_init(full0 + 8 * s, 1); mbar_init(empty0 + 8 * s, 1); }
    mbar_init(done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(Cf::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  for (int i = tid; i < BN; i += NTHR) bias_s[i] = (bias != nullptr && n0 + i < N) ? bf2f(bias[n0 + i]) : 0.f;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp == TMA_WARP && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmW) : "memory");
    for (int kt = 0; kt < nk; kt++) {
      const int s = kt % S;
      if (kt >= S) mbar_wait(empty0 + 8 * s, ((uint32_t)(kt / S) & 1u) ^ 1u);
      const uint32_t st = smem_u32(smem + s * Cf::STAGE_BYTES), bar = full0 + 8 * s;
      mbar_expect(bar, Cf::TX);
      tma2d(st, &tmA, kt * BK, m0, bar);
      tma2d(st + Cf::A_BYTES, &tmW, kt * BK, n0, bar);
    }
  } else if (warp == MMA_WARP && lane == 0) {
    for (int kt = 0; kt < nk; kt++) {
      const int s = kt % S;
      mbar_wait(full0 + 8 * s, (uint32_t)(kt / S) & 1u);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t st = smem_u32(smem + s * Cf::STAGE_BYTES);
#pragma unroll
      for (int j = 0; j < BK / 16; j++)
        mma_bf16(tmem, sdesc128(st + 32 * j), sdesc128(st + Cf::A_BYTES + 32 * j), Cf::IDESC, (kt | j) != 0);
      mma_commit(empty0 + 8 * s);
    }
    mma_commit(done_bar);
  } else if (warp < 4) {
    // epilogue (TMEM lanes 32w..32w+31 = tile rows): accumulator + bias -> bf16 -> padded shared
    // tile -> coalesced 16-byte row stores
    mbar_wait(done_bar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    bf16* tile = reinterpret_cast<bf16*>(smem);
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      float v[32];
      if (nk > 0) tmem_ld32(tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)c0, v);
      else {
#pragma unroll
        for (int i = 0; i < 32; i++) v[i] = 0.f;
      }
#pragma unroll
      for (int i = 0; i < 32; i++) v[i] += bias_s[c0 + i];
#pragma unroll
      for (int i = 0; i < 32; i += 8) *reinterpret_cast<uint4*>(tile + tid * Cf::EPI_LD + c0 + i) = pack8(v + i);
    }
    asm volatile("bar.sync 1, 128;" ::: "memory");
    constexpr int CPR = BN / 8;
    const bool vec = (N % 8) == 0;
    for (int e = tid; e < BM * CPR; e += 128) {
      const int r = e / CPR, c = (e % CPR) * 8;
      const int m = m0 + r, n = n0 + c;
      if (m >= M || n >= N) continue;
      const bf16* srcp = tile + r * Cf::EPI_LD + c;
      bf16* dst = C + (long long)m * N + n;
      if (vec) *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(srcp);
      else
        for (int i = 0; i < 8 && n + i < N; i++) dst[i] = srcp[i];
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cf::TMEM_COLS) : "memory");
  }
  orion_signal(sig);
}

template <int BN>
bool prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  bool ok = cudaFuncSetAttribute((const void*)gemm_bf16_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::SMEM) ==
            cudaSuccess;
  if (ok) done.store(1, std::memory_order_release);
  return ok;
}
// Tile width from the shape only (never the SM partition): 128 when that still gives >= one CTA
// per SM of a whole B200, else 64 (twice the CTAs for BERT-base's N = 768 projections).
// 256-wide tiles (the widest UMMA N: most MMA work per staged A tile) when they still give >= 96
// CTAs (BERT's FFN up-projection), else 128 when that gives >= one CTA per SM, else 64.
inline int bn_for(long long M, long long N) {
  if (cdiv(M, BM) * cdiv(N, 256) >= 96) return 256;
  return cdiv(M, BM) * cdiv(N, 128) >= 148 ? 128 : 64;
}

// cuTensorMapEncodeTiled through cudart's driver entry point (liborion does not link libcuda)
typedef CUresult (*encode_fn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                              const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
inline encode_fn encoder() {
  static encode_fn fn = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (encode_fn) nullptr;
    return (encode_fn)p;
  }();
  return fn;
}
// bf16 row-major [rows][K], box {64, box_rows}, 128-byte swizzle, out-of-bounds zero fill
inline bool map_bf16(CUtensorMap* m, const void* base, long long rows, long long K, int box_rows) {
  cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)K * 2};
  cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  return encoder()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace tcb

// =============================================================================== attention
namespace attn {

constexpr int D = 64;          // head dim (BERT-base: 768 / 12)
constexpr int QB = 64;         // queries per CTA (4 warps x 16)
constexpr int NTH = 128;
constexpr int KLD = D + 8;     // padded K row (bf16): conflict-free 4-byte fragment loads

__device__ __forceinline__ void mma16816(float* c, const uint32_t* a, uint32_t b0, uint32_t b1) {
  asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
               : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
               : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

// SN = S / 16 (S <= 128). q, k, v, o: [B, S, ld] bf16 with head h in columns h*D .. h*D+D-1.
template <int SN>
__global__ void __launch_bounds__(NTH) attention_kernel(const bf16* __restrict__ q, const bf16* __restrict__ k, const bf16* __restrict__ v,
                                                       bf16* __restrict__ o, int ld, float scale, OrionSig sig) {
  constexpr int S = SN * 16, NT = S / 8, VLD = S + 8;
  __shared__ __align__(16) bf16 Ks[S * KLD];
  __shared__ __align__(16) bf16 Vt[D * VLD];
  const int b = blockIdx.z, h = blockIdx.y, tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const long long base = (long long)b * S * ld + h * D;
  for (int e = tid; e < S * (D / 8); e += NTH) {   // K rows and V transposed, 16-byte loads
    const int r = e / (D / 8), c = (e % (D / 8)) * 8;
    *reinterpret_cast<uint4*>(Ks + r * KLD + c) = __ldg(reinterpret_cast<const uint4*>(k + base + (long long)r * ld + c));
    const uint4 u = __ldg(reinterpret_cast<const uint4*>(v + base + (long long)r * ld + c));
    const bf16* e8 = reinterpret_cast<const bf16*>(&u);
#pragma unroll
    for (int i = 0; i < 8; i++) Vt[(c + i) * VLD + r] = e8[i];
  }
  __syncthreads();
  const int q0 = blockIdx.x * QB + warp * 16;
  if (q0 < S) {
    const int g = lane >> 2, t = lane & 3;
    // Q fragments for the 4 K steps over d
    uint32_t qa[D / 16][4];
    const bf16* qr0 = q + base + (long long)(q0 + g) * ld;
    const bf16* qr1 = qr0 + 8LL * ld;
#pragma unroll
    for (int kk = 0; kk < D / 16; kk++) {
      qa[kk][0] = __ldg(reinterpret_cast<const uint32_t*>(qr0 + 16 * kk + 2 * t));
      qa[kk][1] = __ldg(reinterpret_cast<const uint32_t*>(qr1 + 16 * kk + 2 * t));
      qa[kk][2] = __ldg(reinterpret_cast<const uint32_t*>(qr0 + 16 * kk + 8 + 2 * t));
      qa[kk][3] = __ldg(reinterpret_cast<const uint32_t*>(qr1 + 16 * kk + 8 + 2 * t));
    }
    // scores: rows g (c0, c1) and g + 8 (c2, c3), keys 8j + 2t, +1
    float sc[NT][4];
#pragma unroll
    for (int j = 0; j < NT; j++) {
      sc[j][0] = sc[j][1] = sc[j][2] = sc[j][3] = 0.f;
      const bf16* kr = Ks + (8 * j + g) * KLD + 2 * t;
#pragma unroll
      for (int kk = 0; kk < D / 16; kk++)
        mma16816(sc[j], qa[kk], *reinterpret_cast<const uint32_t*>(kr + 16 * kk), *reinterpret_cast<const uint32_t*>(kr + 16 * kk + 8));
    }
    // softmax over keys in fp32: the row's values live in the 4 lanes of a quad
    float mx0 = -FLT_MAX, mx1 = -FLT_MAX;
#pragma unroll
    for (int j = 0; j < NT; j++) {
#pragma unroll
      for (int i = 0; i < 4; i++) sc[j][i] *= scale;
      mx0 = fmaxf(mx0, fmaxf(sc[j][0], sc[j][1]));
      mx1 = fmaxf(mx1, fmaxf(sc[j][2], sc[j][3]));
    }
    mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, 1)); mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, 2));
    mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, 1)); mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, 2));
    float s0 = 0.f, s1 = 0.f;
#pragma unroll
    for (int j = 0; j < NT; j++) {
      sc[j][0] = expf(sc[j][0] - mx0); sc[j][1] = expf(sc[j][1] - mx0);
      sc[j][2] = expf(sc[j][2] - mx1); sc[j][3] = expf(sc[j][3] - mx1);
      s0 += sc[j][0] + sc[j][1];
      s1 += sc[j][2] + sc[j][3];
    }
    s0 += __shfl_xor_sync(0xffffffffu, s0, 1); s0 += __shfl_xor_sync(0xffffffffu, s0, 2);
    s1 += __shfl_xor_sync(0xffffffffu, s1, 1); s1 += __shfl_xor_sync(0xffffffffu, s1, 2);
    // O = P V with P (bf16) taken straight from the score accumulators (C layout == A layout)
    float oc[D / 8][4];
#pragma unroll
    for (int jd = 0; jd < D / 8; jd++) oc[jd][0] = oc[jd][1] = oc[jd][2] = oc[jd][3] = 0.f;
#pragma unroll
    for (int kk = 0; kk < SN; kk++) {
      uint32_t pa[4];
      pa[0] = pack_bf2(sc[2 * kk][0], sc[2 * kk][1]);
      pa[1] = pack_bf2(sc[2 * kk][2], sc[2 * kk][3]);
      pa[2] = pack_bf2(sc[2 * kk + 1][0], sc[2 * kk + 1][1]);
      pa[3] = pack_bf2(sc[2 * kk + 1][2], sc[2 * kk + 1][3]);
#pragma unroll
      for (int jd = 0; jd < D / 8; jd++) {
        const bf16* vr = Vt + (8 * jd + g) * VLD + 16 * kk + 2 * t;
        mma16816(oc[jd], pa, *reinterpret_cast<const uint32_t*>(vr), *reinterpret_cast<const uint32_t*>(vr + 8));
      }
    }
    const float r0 = 1.f / s0, r1 = 1.f / s1;
    bf16* or0 = o + base + (long long)(q0 + g) * ld;
    bf16* or1 = or0 + 8LL * ld;
#pragma unroll
    for (int jd = 0; jd < D / 8; jd++) {
      *reinterpret_cast<uint32_t*>(or0 + 8 * jd + 2 * t) = pack_bf2(oc[jd][0] * r0, oc[jd][1] * r0);
      *reinterpret_cast<uint32_t*>(or1 + 8 * jd + 2 * t) = pack_bf2(oc[jd][2] * r1, oc[jd][3] * r1);
    }
  }
  orion_signal(sig);
}

}  // namespace attn

// ====================================================================== memory-bound bf16 ops
constexpr int TB = 256;
constexpr unsigned MAX_CTAS = 148 * 8;

void vec_geom(LaunchGeom* g, uint64_t n_vec, const void* f) {
  uint64_t ctas = cdiv(n_vec ? n_vec : 1, TB);
  g->grid = dim3((unsigned)(ctas < MAX_CTAS ? ctas : MAX_CTAS));
  g->block = dim3(TB);
  g->smem = 0;
  g->func = f;
}

// LayerNorm over rows of C (C % 8 == 0, C <= 2048): one warp per row, values kept in registers,
// mean then variance of (x - mean) by fixed xor-shuffle trees, fp32; y rounded once to bf16.
constexpr int LN_MAXCH = 8;   // 16-byte chunks per lane
__global__ void __launch_bounds__(TB) layernorm_kernel(const bf16* __restrict__ x, bf16* __restrict__ y, const bf16* __restrict__ gamma,
                                                      const bf16* __restrict__ beta, long long rows, int C, float eps, OrionSig sig) {
  const int lane = threadIdx.x % 32;
  const long long row = (long long)blockIdx.x * (TB / 32) + threadIdx.x / 32;
  if (row < rows) {
    const int nch = C / 8;
    const uint4* xr = reinterpret_cast<const uint4*>(x + row * C);
    float v[LN_MAXCH][8];
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < LN_MAXCH; i++) {
      const int ch = lane + 32 * i;
      if (ch < nch) {
        unpack8(__ldg(xr + ch), v[i]);
#pragma unroll
        for (int e = 0; e < 8; e++) s += v[i][e];
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float mean = s / (float)C;
    float q = 0.f;
#pragma unroll
    for (int i = 0; i < LN_MAXCH; i++) {
      if (lane + 32 * i < nch) {
#pragma unroll
        for (int e = 0; e < 8; e++) { const float d = v[i][e] - mean; q += d * d; }
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    const float rstd = 1.f / sqrtf(q / (float)C + eps);
    uint4* yr = reinterpret_cast<uint4*>(y + row * C);
#pragma unroll
    for (int i = 0; i < LN_MAXCH; i++) {
      const int ch = lane + 32 * i;
      if (ch < nch) {
        float gm[8], bt[8], out[8];
        unpack8(__ldg(reinterpret_cast<const uint4*>(gamma) + ch), gm);
        unpack8(__ldg(reinterpret_cast<const uint4*>(beta) + ch), bt);
#pragma unroll
        for (int e = 0; e < 8; e++) out[e] = (v[i][e] - mean) * rstd * gm[e] + bt[e];
        yr[ch] = pack8(out);
      }
    }
  }
  orion_signal(sig);
}

// GELU (erf form) and residual add: n % 8 == 0, 16-byte aligned
__global__ void __launch_bounds__(TB) gelu_kernel(const bf16* __restrict__ x, bf16* __restrict__ y, long long n8, OrionSig sig) {
  for (long long i = (long long)blockIdx.x * TB + threadIdx.x; i < n8; i += (long long)gridDim.x * TB) {
    float f[8];
    unpack8(__ldg(reinterpret_cast<const uint4*>(x) + i), f);
#pragma unroll
    for (int e = 0; e < 8; e++) f[e] = 0.5f * f[e] * (1.f + erff(f[e] * 0.70710678118654752f));
    reinterpret_cast<uint4*>(y)[i] = pack8(f);
  }
  orion_signal(sig);
}

__global__ void __launch_bounds__(TB) add_bf16_kernel(const bf16* __restrict__ a, const bf16* __restrict__ b, bf16* __restrict__ c,
                                                     long long n8, OrionSig sig) {
  for (long long i = (long long)blockIdx.x * TB + threadIdx.x; i < n8; i += (long long)gridDim.x * TB) {
    float f[8], g[8];
    unpack8(__ldg(reinterpret_cast<const uint4*>(a) + i), f);
    unpack8(__ldg(reinterpret_cast<const uint4*>(b) + i), g);
#pragma unroll
    for (int e = 0; e < 8; e++) f[e] += g[e];
    reinterpret_cast<uint4*>(c)[i] = pack8(f);
  }
  orion_signal(sig);
}

// Embedding gather-sum: out[b, s, :] = word[ids[b, s]] + type[0] + pos[s] (H % 8 == 0)
__global__ void __launch_bounds__(TB) embed_kernel(const int* __restrict__ ids, const bf16* __restrict__ word, const bf16* __restrict__ pos,
                                                  const bf16* __restrict__ typ, bf16* __restrict__ out, int S, int H, long long total8,
                                                  int vocab, OrionSig sig) {
  const int hc = H / 8;
  for (long long i = (long long)blockIdx.x * TB + threadIdx.x; i < total8; i += (long long)gridDim.x * TB) {
    const long long r = i / hc;
    const int c = (int)(i % hc);
    const int s = (int)(r % S);
    int id = __ldg(ids + r);
    id = id < 0 ? 0 : (id >= vocab ? vocab - 1 : id);   // out-of-range ids clamp (documented in orion_kernels.h)
    float w[8], p[8], t[8];
    unpack8(__ldg(reinterpret_cast<const uint4*>(word + (long long)id * H) + c), w);
    unpack8(__ldg(reinterpret_cast<const uint4*>(pos + (long long)s * H) + c), p);
    unpack8(__ldg(reinterpret_cast<const uint4*>(typ) + c), t);
#pragma unroll
    for (int e = 0; e < 8; e++) w[e] = (w[e] + t[e]) + p[e];
    reinterpret_cast<uint4*>(out)[i] = pack8(w);
  }
  orion_signal(sig);
}

// =============================================================================== maxpool bwd
// MaxPool 3x3 / stride 2 / pad 1 backward, gather form. Thread per (n, 2x2 block of inputs rows
// 2a..2a+1, cols 2b..2b+1, 4 channels): the windows that can select those inputs are p in {a, a+1},
// q in {b, b+1}; each window's first maximum (row-major, strict >) is computed once and its dy is
// added to the owned input it selects, windows visited in ascending (p, q) -- the same per-input
// order as a thread per input, so results are bit-identical to that form, with ~9 instead of ~20
// 128-bit window loads per input (round 2's thread per input recomputed every window it shares).
__global__ void __launch_bounds__(TB) maxpool_bwd_kernel(const float* __restrict__ x, const float* __restrict__ dy, float* __restrict__ dx,
                                                        int N, int H, int W, int C, int P, int Q, OrionSig sig) {
  const int C4 = C / 4, HB = (H + 1) / 2, WB = (W + 1) / 2;
  const long long total = (long long)N * HB * WB * C4;
  for (long long i = (long long)blockIdx.x * TB + threadIdx.x; i < total; i += (long long)gridDim.x * TB) {
    const int c = (int)(i % C4) * 4;
    long long t = i / C4;
    const int b = (int)(t % WB); t /= WB;
    const int a = (int)(t % HB);
    const int n = (int)(t / HB);
    float acc[2][2][4];
#pragma unroll
    for (int u = 0; u < 2; u++)
#pragma unroll
      for (int v = 0; v < 2; v++)
#pragma unroll
        for (int e = 0; e < 4; e++) acc[u][v][e] = 0.f;
#pragma unroll
    for (int dp = 0; dp < 2; dp++) {
      const int p = a + dp;
      if (p >= P) continue;
#pragma unroll
      for (int dq = 0; dq < 2; dq++) {
        const int q = b + dq;
        if (q >= Q) continue;
        float best[4] = {-FLT_MAX, -FLT_MAX, -FLT_MAX, -FLT_MAX};
        int arg[4] = {-1, -1, -1, -1};
        bool started = false;
#pragma unroll
        for (int u = 0; u < 3; u++) {
          const int hh = 2 * p - 1 + u;
          if ((unsigned)hh >= (unsigned)H) continue;
#pragma unroll
          for (int vv = 0; vv < 3; vv++) {
            const int ww = 2 * q - 1 + vv;
            if ((unsigned)ww >= (unsigned)W) continue;
            const float4 xv = __ldg(reinterpret_cast<const float4*>(x + (((long long)n * H + hh) * W + ww) * C + c));
            const float xs[4] = {xv.x, xv.y, xv.z, xv.w};
            const int code = u * 3 + vv;
#pragma unroll
            for (int e = 0; e < 4; e++)
              if (!started || xs[e] > best[e]) { best[e] = xs[e]; arg[e] = code; }
            started = true;
          }
        }
        const float4 g = __ldg(reinterpret_cast<const float4*>(dy + (((long long)n * P + p) * Q + q) * C + c));
        const float gs[4] = {g.x, g.y, g.z, g.w};
        // window tap (u, vv) is input (2p-1+u, 2q-1+vv) = owned (2a + ou, 2b + ov) with
        // ou = 2 dp - 1 + u, ov = 2 dq - 1 + vv in {0, 1}
#pragma unroll
        for (int e = 0; e < 4; e++) {
          const int ou = 2 * dp - 1 + arg[e] / 3, ov = 2 * dq - 1 + arg[e] % 3;
#pragma unroll
          for (int u = 0; u < 2; u++)
#pragma unroll
            for (int v = 0; v < 2; v++)
              if (ou == u && ov == v) acc[u][v][e] += gs[e];
        }
      }
    }
#pragma unroll
    for (int u = 0; u < 2; u++) {
      const int h = 2 * a + u;
      if (h >= H) continue;
#pragma unroll
      for (int v = 0; v < 2; v++) {
        const int w = 2 * b + v;
        if (w >= W) continue;
        *reinterpret_cast<float4*>(dx + (((long long)n * H + h) * W + w) * C + c) = make_float4(acc[u][v][0], acc[u][v][1], acc[u][v][2], acc[u][v][3]);
      }
    }
  }
  orion_signal(sig);
}

// =============================================================================== col2im (fp32)
// dx[n,h,w,c] = sum over taps (r, s) with h = p*stride - pad + r, w = q*stride - pad + s (p, q in
// range) of col[(n,p,q)][(r,s,c)]: the second half of a strided convolution's data gradient
// (col = dy W is a dense GEMM). Thread per (n, h, w, 4 channels); taps visited in (r, s) order.
__global__ void __launch_bounds__(TB) col2im_kernel(const float* __restrict__ col, float* __restrict__ dx, int N, int H, int W, int C, int R,
                                                   int S, int st, int pad, int P, int Q, OrionSig sig) {
  const int C4 = C / 4;
  const long long total = (long long)N * H * W * C4;
  const long long rsc = (long long)R * S * C;
  for (long long i = (long long)blockIdx.x * TB + threadIdx.x; i < total; i += (long long)gridDim.x * TB) {
    const int c = (int)(i % C4) * 4;
    long long t = i / C4;
    const int w = (int)(t % W); t /= W;
    const int h = (int)(t % H);
    const int n = (int)(t / H);
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int r = 0; r < R; r++) {
      const int ph = h + pad - r;
      if (ph < 0 || ph % st) continue;
      const int p = ph / st;
      if (p >= P) continue;
      for (int s = 0; s < S; s++) {
        const int pw = w + pad - s;
        if (pw < 0 || pw % st) continue;
        const int q = pw / st;
        if (q >= Q) continue;
        const float4 v = __ldg(reinterpret_cast<const float4*>(col + (((long long)n * P + p) * Q + q) * rsc + ((long long)r * S + s) * C + c));
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
      }
    }
    *reinterpret_cast<float4*>(dx + (((long long)n * H + h) * W + w) * C + c) = acc;
  }
  orion_signal(sig);
}

inline bool al16(uint64_t p) { return (p & 15) == 0; }

}  // namespace

// ================================================================================ table entries
// gemm_bf16: args A, W, C, bias (0 = none), M, N, K
int gemm_bf16_geom(const uint64_t* a, LaunchGeom* g) {
  const long long M = (long long)a[4], N = (long long)a[5], K = (long long)a[6];
  if (M <= 0 || N <= 0 || K <= 0 || (K % 8) != 0 || !al16(a[0]) || !al16(a[1]) || !al16(a[2])) return ORION_E_INVAL;
  if (tcb::encoder() == nullptr) return ORION_E_CUDA;
  const int bn = tcb::bn_for(M, N);
  g->grid = dim3((unsigned)cdiv(N, bn), (unsigned)cdiv(M, tcb::BM));
  g->block = dim3(tcb::NTHR);
  if (bn == 256) {
    if (!tcb::prepare<256>()) return ORION_E_CUDA;
    g->smem = tcb::Cfg<256>::SMEM; g->func = (const void*)tcb::gemm_bf16_kernel<256>; g->pipe = ORION_PIPE_BF16;
  } else if (bn == 128) {
    if (!tcb::prepare<128>()) return ORION_E_CUDA;
    g->smem = tcb::Cfg<128>::SMEM; g->func = (const void*)tcb::gemm_bf16_kernel<128>; g->pipe = ORION_PIPE_BF16;
  } else {
    if (!tcb::prepare<64>()) return ORION_E_CUDA;
    g->smem = tcb::Cfg<64>::SMEM; g->func = (const void*)tcb::gemm_bf16_kernel<64>; g->pipe = ORION_PIPE_BF16;
  }
  return 0;
}
int gemm_bf16_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  const long long M = (long long)a[4], N = (long long)a[5], K = (long long)a[6];
  const int bn = g.func == (const void*)tcb::gemm_bf16_kernel<256> ? 256 : g.func == (const void*)tcb::gemm_bf16_kernel<128> ? 128 : 64;
  CUtensorMap ma, mw;
  if (!tcb::map_bf16(&ma, (const void*)a[0], M, K, tcb::BM) || !tcb::map_bf16(&mw, (const void*)a[1], N, K, bn))
    return ORION_E_CUDA;
  if (bn == 256)
    tcb::gemm_bf16_kernel<256><<<g.grid, g.block, g.smem, s>>>(ma, mw, (bf16*)a[2], (const bf16*)a[3], (int)M, (int)N, (int)K, sig);
  else if (bn == 128)
    tcb::gemm_bf16_kernel<128><<<g.grid, g.block, g.smem, s>>>(ma, mw, (bf16*)a[2], (const bf16*)a[3], (int)M, (int)N, (int)K, sig);
  else
    tcb::gemm_bf16_kernel<64><<<g.grid, g.block, g.smem, s>>>(ma, mw, (bf16*)a[2], (const bf16*)a[3], (int)M, (int)N, (int)K, sig);
  CHECK_LAUNCH();
}

// attention: args q, k, v, o, B, S, heads, head_dim, ld
static const void* attn_fn(int sn) {
  switch (sn) {
    case 1: return (const void*)attn::attention_kernel<1>;
    case 2: return (const void*)attn::attention_kernel<2>;
    case 4: return (const void*)attn::attention_kernel<4>;
    case 8: return (const void*)attn::attention_kernel<8>;
    default: return nullptr;
  }
}
int attention_geom(const uint64_t* a, LaunchGeom* g) {
  const long long B = (long long)a[4], S = (long long)a[5], heads = (long long)a[6], d = (long long)a[7], ld = (long long)a[8];
  if (B <= 0 || heads <= 0 || d != attn::D || S % 16 != 0 || ld < heads * d || (ld % 8) != 0) return ORION_E_INVAL;
  const void* f = attn_fn((int)(S / 16));
  if (!f || !al16(a[0]) || !al16(a[1]) || !al16(a[2]) || !al16(a[3])) return ORION_E_INVAL;
  g->grid = dim3((unsigned)cdiv(S, attn::QB), (unsigned)heads, (unsigned)B);
  g->block = dim3(attn::NTH);
  g->smem = 0;
  g->func = f;
  g->pipe = ORION_PIPE_BF16;   // QK^T and PV on mma.sync bf16 (tensor pipe)
  return 0;
}
int attention_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  auto q = (const bf16*)a[0]; auto k = (const bf16*)a[1]; auto v = (const bf16*)a[2]; auto o = (bf16*)a[3];
  const int ld = (int)a[8];
  const float scale = 1.f / sqrtf((float)a[7]);
  switch ((int)a[5] / 16) {
    case 1: attn::attention_kernel<1><<<g.grid, g.block, 0, s>>>(q, k, v, o, ld, scale, sig); break;
    case 2: attn::attention_kernel<2><<<g.grid, g.block, 0, s>>>(q, k, v, o, ld, scale, sig); break;
    case 4: attn::attention_kernel<4><<<g.grid, g.block, 0, s>>>(q, k, v, o, ld, scale, sig); break;
    default: attn::attention_kernel<8><<<g.grid, g.block, 0, s>>>(q, k, v, o, ld, scale, sig); break;
  }
  CHECK_LAUNCH();
}

// layernorm: args x, y, gamma, beta, rows, C, eps_bits
int layernorm_geom(const uint64_t* a, LaunchGeom* g) {
  const long long rows = (long long)a[4], C = (long long)a[5];
  if (rows <= 0 || C <= 0 || C % 8 != 0 || C > 8 * 32 * LN_MAXCH) return ORION_E_INVAL;
  if (!al16(a[0]) || !al16(a[1]) || !al16(a[2]) || !al16(a[3])) return ORION_E_INVAL;
  g->grid = dim3((unsigned)cdiv(rows, TB / 32)); g->block = dim3(TB); g->smem = 0; g->func = (const void*)layernorm_kernel;
  return 0;
}
int layernorm_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  layernorm_kernel<<<g.grid, g.block, 0, s>>>((const bf16*)a[0], (bf16*)a[1], (const bf16*)a[2], (const bf16*)a[3], (long long)a[4],
                                              (int)a[5], u2f(a[6]), sig);
  CHECK_LAUNCH();
}

// gelu: args x, y, n ; add_bf16: args a, b, c, n   (n % 8 == 0, 16-byte aligned)
int gelu_geom(const uint64_t* a, LaunchGeom* g) {
  if (a[2] == 0 || a[2] % 8 || !al16(a[0]) || !al16(a[1])) return ORION_E_INVAL;
  vec_geom(g, a[2] / 8, (const void*)gelu_kernel);
  return 0;
}
int gelu_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  gelu_kernel<<<g.grid, g.block, 0, s>>>((const bf16*)a[0], (bf16*)a[1], (long long)(a[2] / 8), sig);
  CHECK_LAUNCH();
}
int add_bf16_geom(const uint64_t* a, LaunchGeom* g) {
  if (a[3] == 0 || a[3] % 8 || !al16(a[0]) || !al16(a[1]) || !al16(a[2])) return ORION_E_INVAL;
  vec_geom(g, a[3] / 8, (const void*)add_bf16_kernel);
  return 0;
}
int add_bf16_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  add_bf16_kernel<<<g.grid, g.block, 0, s>>>((const bf16*)a[0], (const bf16*)a[1], (bf16*)a[2], (long long)(a[3] / 8), sig);
  CHECK_LAUNCH();
}

// embed: args ids, word, pos, type, out, B, S, H, vocab
int embed_geom(const uint64_t* a, LaunchGeom* g) {
  const long long B = (long long)a[5], S = (long long)a[6], H = (long long)a[7];
  if (B <= 0 || S <= 0 || H <= 0 || H % 8 || (long long)a[8] <= 0) return ORION_E_INVAL;
  if (!al16(a[1]) || !al16(a[2]) || !al16(a[3]) || !al16(a[4])) return ORION_E_INVAL;
  vec_geom(g, (uint64_t)(B * S * H / 8), (const void*)embed_kernel);
  return 0;
}
int embed_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  const long long B = (long long)a[5], S = (long long)a[6], H = (long long)a[7];
  embed_kernel<<<g.grid, g.block, 0, s>>>((const int*)a[0], (const bf16*)a[1], (const bf16*)a[2], (const bf16*)a[3], (bf16*)a[4], (int)S,
                                          (int)H, B * S * H / 8, (int)a[8], sig);
  CHECK_LAUNCH();
}

// maxpool_bwd: args x, dy, dx, N, H, W, C, P, Q   (C % 4 == 0)
int maxpool_bwd_geom(const uint64_t* a, LaunchGeom* g) {
  const long long N = (long long)a[3], H = (long long)a[4], W = (long long)a[5], C = (long long)a[6];
  if (N <= 0 || H <= 0 || W <= 0 || C <= 0 || C % 4 || !al16(a[0]) || !al16(a[1]) || !al16(a[2])) return ORION_E_INVAL;
  if ((long long)a[7] != (H - 1) / 2 + 1 || (long long)a[8] != (W - 1) / 2 + 1) return ORION_E_INVAL;
  vec_geom(g, (uint64_t)(N * ((H + 1) / 2) * ((W + 1) / 2) * C / 4), (const void*)maxpool_bwd_kernel);
  // up to 8 resident waves instead of one: at ResNet's training batch the op runs ~0.3 ms, and a
  // non-preemptible BE kernel's CTAs would each hold their SM that long against an arriving HP
  // request; shorter-lived CTAs free SMs as they retire (grid-stride loop, results do
  // not depend on the grid)
  const uint64_t ctas = cdiv((uint64_t)(N * ((H + 1) / 2) * ((W + 1) / 2) * C / 4), TB);
  g->grid = dim3((unsigned)(ctas < 8ull * MAX_CTAS ? ctas : 8ull * MAX_CTAS));
  return 0;
}
int maxpool_bwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  maxpool_bwd_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (float*)a[2], (int)a[3], (int)a[4], (int)a[5],
                                                (int)a[6], (int)a[7], (int)a[8], sig);
  CHECK_LAUNCH();
}

// col2im: args col, dx, N, H, W, C, R, S, stride, pad, P, Q   (C % 4 == 0)
int col2im_geom(const uint64_t* a, LaunchGeom* g) {
  const long long N = (long long)a[2], H = (long long)a[3], W = (long long)a[4], C = (long long)a[5];
  const long long R = (long long)a[6], S = (long long)a[7], st = (long long)a[8], pad = (long long)a[9];
  if (N <= 0 || H <= 0 || W <= 0 || C <= 0 || C % 4 || R <= 0 || S <= 0 || st <= 0 || pad < 0 || !al16(a[0]) || !al16(a[1]))
    return ORION_E_INVAL;
  if ((long long)a[10] != (H + 2 * pad - R) / st + 1 || (long long)a[11] != (W + 2 * pad - S) / st + 1) return ORION_E_INVAL;
  vec_geom(g, (uint64_t)(N * H * W * C / 4), (const void*)col2im_kernel);
  return 0;
}
int col2im_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  col2im_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (int)a[2], (int)a[3], (int)a[4], (int)a[5], (int)a[6], (int)a[7],
                                           (int)a[8], (int)a[9], (int)a[10], (int)a[11], sig);
  CHECK_LAUNCH();
}
