// Weight-gradient GEMM on the tensor cores (gemm flags = 1): C[M][N] = sum_k A[k][m] B[k][n] with
// both operands MN-major in HBM (dy [rows][Cout], x [rows][Cin] of a 1x1 convolution or Linear
// layer), fp32 through 3xTF32 on tcgen05 (x = hi + lo, D += lo.hi + hi.lo + hi.hi).
//
// The streaming FFMA kernel (wgs.cu) reaches HBM speed only while M*N/(M+N) stays small; beyond ~40
// flop/B it is bound by the FFMA issue rate (MobileNetV2's late layers, ResNet's 1x1 convs). Here:
//  * one elected thread streams BK = 32-row stages with 2-D TMA, 128-byte swizzle, straight into
//    the MN-major canonical layout UMMA reads (32-element atoms of 8 k-rows x 128 B; atoms along
//    M / N 4 KB apart = LBO, k-groups 1 KB apart = SBO) -- no transposition anywhere;
//  * four converter warps form lo = x - trunc_tf32(x) in place-shaped copies (elementwise, so the
//    swizzled layout is preserved); the raw fp32 tile serves as hi (the tensor core reads tf32);
//  * one thread issues tcgen05.mma kind::tf32 with transposed (MN-major) A and B descriptors into
//    two TMEM accumulators (main, corrections); the converter warps then read TMEM back;
//  * K is split over CTAs (shape-only count); the fp32 partial tiles are summed in split order (fp64)
//    by a second, many-CTA launch of the op, so results are deterministic and partition-independent.
#include <cmath>
#include <cstdlib>

#include "common.cuh"
#include "tma.cuh"

namespace {
namespace atc {
using namespace tmah;

constexpr int BM = 128, BK = 16, NTHR = 192;   // warps: 0 TMA, 1 MMA + TMEM owner, 2-5 converters / epilogue
// (16-row stages: deep rings -- 6-8 stages -- keep the loads of one CTA per SM in flight)
constexpr int CONV_THREADS = 128;
constexpr int BOX_BYTES = 32 * BK * 4;   // one TMA box: 32 elements (128 B) x BK rows = one MN atom column

#ifndef ATC_MAX_STAGES
#define ATC_MAX_STAGES 8
#endif
constexpr int MAX_STAGES = ATC_MAX_STAGES;   // ring depth cap (small-N tiles: more 16-row stages in flight)
template <int BN_>
struct Cfg {
  static constexpr int BN = BN_;
  static constexpr int A_BYTES = BM * BK * 4, B_BYTES = BN * BK * 4;
  static constexpr int STAGE = 2 * (A_BYTES + B_BYTES);   // [A raw][A lo][B raw][B lo]
  static constexpr int STAGES = (200 * 1024) / STAGE > MAX_STAGES ? MAX_STAGES : (200 * 1024) / STAGE;
  static constexpr int SMEM = STAGES * STAGE + 1024 + 256;
  static constexpr int TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;
  // kind::tf32: D fp32 (bit 4), A, B tf32 (bits 7, 10), A and B MN-major (bits 15, 16), N>>3, M>>4
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | (1u << 16) | ((uint32_t)(BN >> 3) << 17) |
                                    ((uint32_t)(BM >> 4) << 24);
  static constexpr uint32_t TX = A_BYTES + B_BYTES;
};

struct Params {
  int DM, DN, K;      // M side (TMEM lanes), N side, rows
  int trans;          // 0: C[m][n]; 1: C[n][m] (M side = the gemm's N operand)
  float* C;
  long long ldc;
  int tiles_n, tiles, split, kps;
  float* part;        // [tile][split][BM*BN] fp32 partial tiles (split > 1)
  // convolution weight gradient (CONV): rows are blocks of PB x QB output positions of one image;
  // x boxes of column col take tap (col / C) shifted by the stride (4-D TMA, zero fill = padding)
  int cv_C, cv_S, stride, pad, QB, PB, npb, nqb;
};

__device__ __forceinline__ uint64_t desc_mn128(uint32_t addr) {
  // MN-major tf32 operands need the 128-byte swizzle with 32-byte atoms (SWIZZLE_128B_BASE32B,
  // layout type 1; TMA CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B): atoms of 4 k-rows x 128 B (32 tf32
  // along M / N). LBO = BOX_BYTES between MN atoms (one TMA box), SBO = 512 B between 4-row k-groups;
  // version 1 (bit 46). (The 16-byte-granular SWIZZLE_128B layout reads as zeros for MN-major tf32.)
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)(BOX_BYTES >> 4) << 16) | ((uint64_t)(512 >> 4) << 32) | (1ull << 46) | (1ull << 61);
}
__device__ __forceinline__ void mma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
               "l"(a), "l"(b), "r"(idesc), "r"(acc)
               : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t mbar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(mbar) : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]),
        "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]),
        "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]),
        "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}
__device__ __forceinline__ float trunc_tf32(float x) { return __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); }

template <int BN, bool CONV>
__global__ void __launch_bounds__(NTHR, 1) atc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                                                     Params p, OrionSig sig) {
  using C_ = Cfg<BN>;
  constexpr int A_BYTES = C_::A_BYTES, B_BYTES = C_::B_BYTES, STAGE = C_::STAGE, S = C_::STAGES;
  extern __shared__ __align__(1024) unsigned char atc_raw[];
  // 1024-byte alignment for the swizzle atoms, by offsetting the shared array itself (keeps LDS/STS)
  unsigned char* smem = atc_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(atc_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * STAGE);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 * S + 2);
  const uint32_t full0 = smem_u32(bars), conv0 = full0 + 8 * S, empty0 = conv0 + 8 * S, done_bar = empty0 + 8 * S;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int tile = blockIdx.x, z = blockIdx.y;
  const int m0 = (tile / p.tiles_n) * BM, n0 = (tile % p.tiles_n) * BN;
  const int k0 = z * p.kps, k1 = min(p.K, k0 + p.kps);
  const int nst = (k1 - k0 + BK - 1) / BK;

  if (tid == 0) {
    for (int s = 0; s < S; s++) { mbar_init(full0 + 8 * s, 1); mbar_init(conv0 + 8 * s, CONV_THREADS / 32); mbar_init(empty0 + 8 * s, 1); }
    mbar_init(done_bar, 1);
    fence_barrier_init();
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(C_::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // CONV: the tile's box columns are fixed for the whole CTA -- decode each one's (channel, tap
      // offset) once; the position block advances by counters. (Per-stage integer divisions on this
      // single issuing thread made it the bottleneck: 1.4 us per stage, ncu.)
      int ca[BM / 32], qa[BM / 32], pa[BM / 32], cb_[BN / 32], qb_[BN / 32], pb_[BN / 32];
      int qb = 0, pb = 0, nimg = 0;
      if (CONV) {
        auto decode = [&](bool is_x, int col, int& c, int& dq, int& dp) {
          if (!is_x) { c = col; dq = 0; dp = 0; return; }
          const int tap = col / p.cv_C, r = tap / p.cv_S, sx = tap - r * p.cv_S;
          c = col - tap * p.cv_C; dq = sx - p.pad; dp = r - p.pad;
        };
#pragma unroll
        for (int j = 0; j < BM / 32; j++) decode(p.trans != 0, m0 + 32 * j, ca[j], qa[j], pa[j]);
#pragma unroll
        for (int j = 0; j < BN / 32; j++) decode(p.trans == 0, n0 + 32 * j, cb_[j], qb_[j], pb_[j]);
        const int b0 = k0 / BK;
        qb = b0 % p.nqb;
        const int t2 = b0 / p.nqb;
        pb = t2 % p.npb; nimg = t2 / p.npb;
      }
#pragma unroll 1
      for (int it = 0; it < nst; it++) {
        const int s = it % S;
        if (it >= S) mbar_wait(empty0 + 8 * s, ((uint32_t)(it / S) & 1u) ^ 1u);
        const uint32_t st = smem_u32(smem + (size_t)s * STAGE), bar = full0 + 8 * s;
        mbar_expect(bar, C_::TX);
        const int kk = k0 + it * BK;
        if (!CONV) {
#pragma unroll
          for (int j = 0; j < BM / 32; j++) tma_load2d(st + j * BOX_BYTES, &tmA, m0 + 32 * j, kk, bar);
#pragma unroll
          for (int j = 0; j < BN / 32; j++) tma_load2d(st + 2 * A_BYTES + j * BOX_BYTES, &tmB, n0 + 32 * j, kk, bar);
        } else {
          // stage = position block (image nimg, output rows p0.., columns q0..); dy boxes take the
          // block itself, x boxes the block shifted by the tap (zero fill = padding)
          const int p0 = pb * p.PB, q0 = qb * p.QB;
          const int qs = q0 * p.stride, ps = p0 * p.stride;
          const bool ax = p.trans != 0;
#pragma unroll
          for (int j = 0; j < BM / 32; j++)
            tma_load4d(st + j * BOX_BYTES, &tmA, ca[j], ax ? qs + qa[j] : q0, ax ? ps + pa[j] : p0, nimg, bar);
#pragma unroll
          for (int j = 0; j < BN / 32; j++)
            tma_load4d(st + 2 * A_BYTES + j * BOX_BYTES, &tmB, cb_[j], ax ? q0 : qs + qb_[j], ax ? p0 : ps + pb_[j], nimg, bar);
          if (++qb == p.nqb) { qb = 0; if (++pb == p.npb) { pb = 0; ++nimg; } }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t d_main = tmem, d_corr = tmem + BN;
#pragma unroll 1
      for (int it = 0; it < nst; it++) {
        const int s = it % S;
        const uint32_t ph = (uint32_t)(it / S) & 1u;
        mbar_wait(full0 + 8 * s, ph);
        mbar_wait(conv0 + 8 * s, ph);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t st = smem_u32(smem + (size_t)s * STAGE);
        const uint32_t a_hi = st, a_lo = st + A_BYTES, b_hi = st + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
        const uint32_t idesc = C_::IDESC;
#pragma unroll
        for (int ks = 0; ks < BK / 8; ks++) {
          const uint32_t o = ks * 1024;   // next 8 rows (two 4-row atoms) inside every MN atom column
          const uint32_t acc = (it | ks) != 0;
          mma_tf32(d_corr, desc_mn128(a_lo + o), desc_mn128(b_hi + o), idesc, acc);
          mma_tf32(d_corr, desc_mn128(a_hi + o), desc_mn128(b_lo + o), idesc, 1);
          mma_tf32(d_main, desc_mn128(a_hi + o), desc_mn128(b_hi + o), idesc, acc);
        }
        mma_commit(empty0 + 8 * s);
      }
      mma_commit(done_bar);
    }
  } else {
    // ---------------- converters: lo = x - trunc(x), same (swizzled) layout
    const int ct = tid - 64;
#pragma unroll 1
    for (int it = 0; it < nst; it++) {
      const int s = it % S;
      mbar_wait(full0 + 8 * s, (uint32_t)(it / S) & 1u);
      unsigned char* st = smem + (size_t)s * STAGE;
      const float4* ahi = reinterpret_cast<const float4*>(st);
      float4* alo = reinterpret_cast<float4*>(st + A_BYTES);
      constexpr int AQ = A_BYTES / 16 / CONV_THREADS, BQ = B_BYTES / 16 / CONV_THREADS;
      float4 va[AQ], vb[BQ > 0 ? BQ : 1];
#pragma unroll
      for (int j = 0; j < AQ; j++) va[j] = ahi[ct + CONV_THREADS * j];
      const float4* bhi = reinterpret_cast<const float4*>(st + 2 * A_BYTES);
      float4* blo = reinterpret_cast<float4*>(st + 2 * A_BYTES + B_BYTES);
#pragma unroll
      for (int j = 0; j < BQ; j++) vb[j] = bhi[ct + CONV_THREADS * j];
#pragma unroll
      for (int j = 0; j < AQ; j++)
        alo[ct + CONV_THREADS * j] = make_float4(va[j].x - trunc_tf32(va[j].x), va[j].y - trunc_tf32(va[j].y), va[j].z - trunc_tf32(va[j].z),
                                                 va[j].w - trunc_tf32(va[j].w));
#pragma unroll
      for (int j = 0; j < BQ; j++)
        blo[ct + CONV_THREADS * j] = make_float4(vb[j].x - trunc_tf32(vb[j].x), vb[j].y - trunc_tf32(vb[j].y), vb[j].z - trunc_tf32(vb[j].z),
                                                 vb[j].w - trunc_tf32(vb[j].w));
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(conv0 + 8 * s);
    }
    // ---------------- epilogue: TMEM lanes 32 (warp % 4) .. +31 = tile rows; 32 columns at a time
    mbar_wait(done_bar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  }
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  // all TMEM reads happen below (warps 2-5), partial tiles / results written, then dealloc
  float* part = p.part ? p.part + ((long long)tile * p.split + z) * (BM * BN) : nullptr;
  if (warp >= 2) {
    const int q = warp & 3, row = 32 * q + lane, m = m0 + row;
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t mv[32], cv[32];
      const uint32_t base = tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)c0;
      tmem_ld32(base, mv);
      tmem_ld32(base + BN, cv);
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (p.split == 1) {
#pragma unroll
        for (int j = 0; j < 32; j++) {
          const int n = n0 + c0 + j;
          const float v = __uint_as_float(mv[j]) + __uint_as_float(cv[j]);
          if (m < p.DM && n < p.DN) {
            if (p.trans) p.C[(long long)n * p.ldc + m] = v;
            else p.C[(long long)m * p.ldc + n] = v;
          }
        }
      } else {
        float4* dst = reinterpret_cast<float4*>(part + (size_t)row * BN + c0);
#pragma unroll
        for (int j = 0; j < 32; j += 4)
          dst[j / 4] = make_float4(__uint_as_float(mv[j]) + __uint_as_float(cv[j]), __uint_as_float(mv[j + 1]) + __uint_as_float(cv[j + 1]),
                                   __uint_as_float(mv[j + 2]) + __uint_as_float(cv[j + 2]), __uint_as_float(mv[j + 3]) + __uint_as_float(cv[j + 3]));
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C_::TMEM_COLS) : "memory");
  }
  if (p.split == 1) orion_signal(sig);   // else the combine kernel below signals
}

// Ordered combine of the split partials (a second launch of the op, many CTAs: the serial last-CTA
// combine of round 2's first version cost ~25 us per launch): thread = 4 consecutive elements of
// one tile, partials added in split order in fp64 with 8 splits' loads in flight; writes C.
constexpr int CMB_THREADS = 256;
template <int BN>
__global__ void __launch_bounds__(CMB_THREADS) atc_combine_kernel(Params p, OrionSig sig) {
  constexpr int V = BM * BN, V4 = V / 4, per_tile = (V4 + CMB_THREADS - 1) / CMB_THREADS;
  const int tile = blockIdx.x / per_tile;
  const int v4 = (blockIdx.x % per_tile) * CMB_THREADS + threadIdx.x;
  if (v4 < V4) {
    const float4* src = reinterpret_cast<const float4*>(p.part + (long long)tile * p.split * V) + v4;
    double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
    int z = 0;
    for (; z + 7 < p.split; z += 8) {
      float4 t[8];
#pragma unroll
      for (int i = 0; i < 8; i++) t[i] = __ldcg(src + (long long)(z + i) * V4);
#pragma unroll
      for (int i = 0; i < 8; i++) { a0 += t[i].x; a1 += t[i].y; a2 += t[i].z; a3 += t[i].w; }
    }
    for (; z < p.split; z++) {
      const float4 t = __ldcg(src + (long long)z * V4);
      a0 += t.x; a1 += t.y; a2 += t.z; a3 += t.w;
    }
    const int m0 = (tile / p.tiles_n) * BM, n0 = (tile % p.tiles_n) * BN;
    const int v = 4 * v4, m = m0 + v / BN, nb = n0 + v % BN;
    const double a[4] = {a0, a1, a2, a3};
#pragma unroll
    for (int j = 0; j < 4; j++) {
      const int n = nb + j;
      if (m < p.DM && n < p.DN) {
        if (p.trans) p.C[(long long)n * p.ldc + m] = (float)a[j];
        else p.C[(long long)m * p.ldc + n] = (float)a[j];
      }
    }
  }
  orion_signal(sig);
}

struct Plan { int trans, bn, tiles_n, tiles, split, kps; };

inline int bn_for(long long DN) { return DN <= 32 ? 32 : DN <= 64 ? 64 : 128; }   // BN <= 128: >= 6 stages

inline Plan plan(long long M, long long N, long long K) {
  Plan best{};
  double best_cost = 1e300;
  for (int trans = 0; trans < 2; trans++) {
    const long long DM = trans ? N : M, DN = trans ? M : N;
    const int bn = bn_for(DN);
    const long long tm = cdiv(DM, BM), tn = cdiv(DN, bn), tiles = tm * tn;
    const double padded = (double)tiles * BM * bn;   // tensor work (and smem traffic) per row
    if (padded < best_cost) {
      best_cost = padded;
      best.trans = trans; best.bn = bn; best.tiles_n = (int)tn; best.tiles = (int)tiles;
    }
  }
  // split K so that the streaming time per CTA (operand bytes / CTAs) and the serial ordered combine
  // of a tile's partials (split x tile bytes, read by its last CTAs) balance: split ~ sqrt(operand
  // bytes / (tiles x tile bytes)), at most one CTA per SM of a 148-SM part (~200 KB of stages each)
  // one CTA per SM of a 148-SM part (~200 KB of stages each); the partial tiles (written once,
  // read once by the parallel combine) stay within the operand bytes
  const double ob = 4.0 * (double)K * (double)(M + N), tb = 4.0 * BM * best.bn;
  long long split = (long long)(ob / (2.0 * (double)best.tiles * tb));
  const long long smax = best.tiles >= 148 ? 1 : 148 / best.tiles;
  if (split > smax) split = smax;
  if (split < 1) split = 1;
  const long long kmax = K / (4LL * BK);                         // >= 4 stages per split
  if (split > kmax) split = kmax > 0 ? kmax : 1;
  // accuracy: the tensor core accumulates a split's rows in fp32 inside TMEM; chains of <= 2048 rows
  // keep 3xTF32 within the single-op bound (rel 1e-5; one K = 4704 chain measured 1.13e-5), the
  // splits themselves are added in fp64
  const long long kchain = (K + 2047) / 2048;
  if (split < kchain) split = kchain;
  if (split > 1024) split = 1024;
  best.kps = (int)(cdiv(cdiv(K, split), BK) * BK);
  best.split = (int)cdiv(K, best.kps);
  return best;
}

inline uint64_t ws_bytes(const Plan& p) {
  if (p.split <= 1) return 0;
  const uint64_t V = (uint64_t)BM * p.bn;
  return WS_TICKET_BYTES + (uint64_t)p.tiles * p.split * V * 4;
}
inline unsigned combine_ctas(const Plan& p) { return (unsigned)(p.tiles * cdiv((uint64_t)BM * p.bn / 4, CMB_THREADS)); }

template <int BN, bool CONV>
bool prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  if (cudaFuncSetAttribute((const void*)atc_kernel<BN, CONV>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::SMEM) != cudaSuccess) {
    (void)cudaGetLastError();
    return false;
  }
  done.store(1, std::memory_order_release);
  return true;
}

inline const void* fn_of(int bn, bool conv = false) {
  switch (bn) {
    case 32: return conv ? (const void*)atc_kernel<32, true> : (const void*)atc_kernel<32, false>;
    case 64: return conv ? (const void*)atc_kernel<64, true> : (const void*)atc_kernel<64, false>;
    default: return conv ? (const void*)atc_kernel<128, true> : (const void*)atc_kernel<128, false>;
  }
}
inline int smem_of(int bn) {
  switch (bn) {
    case 32: return Cfg<32>::SMEM;
    case 64: return Cfg<64>::SMEM;
    default: return Cfg<128>::SMEM;
  }
}
inline bool prepare_of(int bn, bool conv = false) {
  switch (bn) {
    case 32: return conv ? prepare<32, true>() : prepare<32, false>();
    case 64: return conv ? prepare<64, true>() : prepare<64, false>();
    default: return conv ? prepare<128, true>() : prepare<128, false>();
  }
}

// launch the tile kernel (+ the ordered combine when split > 1)
template <bool CONV>
int launch_pair(const LaunchGeom& g, const Plan& pl, const CUtensorMap& mA, const CUtensorMap& mB, const Params& p, OrionSig sig,
                cudaStream_t s) {
  const OrionSig none{nullptr, nullptr, 0, 0};
  const OrionSig s1 = pl.split > 1 ? none : sig;   // split > 1: the combine kernel signals
  switch (pl.bn) {
    case 32: atc_kernel<32, CONV><<<g.grid, g.block, g.smem, s>>>(mA, mB, p, s1); break;
    case 64: atc_kernel<64, CONV><<<g.grid, g.block, g.smem, s>>>(mA, mB, p, s1); break;
    default: atc_kernel<128, CONV><<<g.grid, g.block, g.smem, s>>>(mA, mB, p, s1); break;
  }
  if (pl.split > 1) {
    const unsigned cg = combine_ctas(pl);
    switch (pl.bn) {
      case 32: atc_combine_kernel<32><<<cg, CMB_THREADS, 0, s>>>(p, sig); break;
      case 64: atc_combine_kernel<64><<<cg, CMB_THREADS, 0, s>>>(p, sig); break;
      default: atc_combine_kernel<128><<<cg, CMB_THREADS, 0, s>>>(p, sig); break;
    }
  }
  return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
}

// ---- convolution weight gradient: dW[K][R][S][C] = sum over (n, p, q) of dy[n,p,q,k] x-window
struct ConvGeo { int N, H, W, C, K, R, S, stride, pad, P, Q; };
inline void conv_blocks(const ConvGeo& c, int& QB, int& PB, int& npb, int& nqb) {
  // 16 positions per stage: QB x PB with the least zero-filled padding of the P x Q grid
  double best = 1e30;
  for (int qb = 16; qb >= 1; qb /= 2) {
    const int pb = BK / qb;
    const double w = (double)cdiv(c.Q, qb) * qb * cdiv(c.P, pb) * pb;
    if (w < best - 1e-9) { best = w; QB = qb; PB = pb; }
  }
  npb = (int)cdiv(c.P, PB);
  nqb = (int)cdiv(c.Q, QB);
}
inline Plan plan_conv(const ConvGeo& c) {
  int QB, PB, npb, nqb;
  conv_blocks(c, QB, PB, npb, nqb);
  const long long rows = (long long)c.N * npb * nqb * BK;
  const long long RSC = (long long)c.R * c.S * c.C;
  Plan best{};
  double best_cost = 1e300;
  for (int trans = 0; trans < 2; trans++) {
    const long long DM = trans ? RSC : c.K, DN = trans ? c.K : RSC;
    const int bn = bn_for(DN);
    const long long tm = cdiv(DM, BM), tn = cdiv(DN, bn), tiles = tm * tn;
    const double padded = (double)tiles * BM * bn;
    if (padded < best_cost) { best_cost = padded; best.trans = trans; best.bn = bn; best.tiles_n = (int)tn; best.tiles = (int)tiles; }
  }
  const double ob = 4.0 * (double)c.N * c.P * c.Q * (double)(c.K + RSC), tb = 4.0 * BM * best.bn;
  long long split = (long long)(ob / (2.0 * (double)best.tiles * tb));
  const long long smax = best.tiles >= 148 ? 1 : 148 / best.tiles;
  if (split > smax) split = smax;
  if (split < 1) split = 1;
  const long long kmax = rows / (4LL * BK);
  if (split > kmax) split = kmax > 0 ? kmax : 1;
  const long long kchain = (rows + 2047) / 2048;
  if (split < kchain) split = kchain;
  if (split > 1024) split = 1024;
  best.kps = (int)(cdiv(cdiv(rows, split), BK) * BK);
  best.split = (int)cdiv(rows, best.kps);
  return best;
}

}  // namespace atc
}  // namespace

// ---- entry points used by gemm.cu (flags = 1 routing): the tensor path for weight gradients whose
// FFMA streaming form is compute-bound, i.e. M*N/(M+N) >= ATC_MIN_INTENSITY (flop per byte / 2)
static int atc_min_intensity() {
  static const int v = [] {
    const char* e = getenv("ORION_ATC_MIN_AI");   // tuning knob (shape routing only)
    return e ? atoi(e) : 40;
  }();
  return v;
}

uint64_t atc_ws_bytes(long long M, long long N, long long K) {
  if (M <= 0 || N <= 0 || K <= 0) return 0;
  return atc::ws_bytes(atc::plan(M, N, K));
}

bool atc_try_geom(const uint64_t* a, LaunchGeom* g) {
  const long long M = a[4], N = a[5], K = a[6], lda = a[7], ldb = a[8];
  if ((int)a[10] != 1 || a[3] != 0) return false;
  if (M * N < (long long)atc_min_intensity() * (M + N)) return false;
  if (K < 4 * atc::BK || lda % 4 || ldb % 4 || M % 4 || N % 4) return false;
  if (!tmah::al16((const void*)a[0]) || !tmah::al16((const void*)a[1]) || tmah::encoder() == nullptr) return false;
  if (M >= (1LL << 24) || N >= (1LL << 24) || K >= (1LL << 31)) return false;
  atc::Plan pl = atc::plan(M, N, K);
  if (pl.split > 1 && (a[11] == 0 || a[12] < atc::ws_bytes(pl))) return false;
  if (!atc::prepare_of(pl.bn)) return false;
  g->grid = dim3((unsigned)pl.tiles, (unsigned)pl.split);
  g->sig_ctas = pl.split > 1 ? atc::combine_ctas(pl) : 0;
  g->block = dim3(atc::NTHR);
  g->smem = atc::smem_of(pl.bn);
  g->func = atc::fn_of(pl.bn);
  g->pipe = ORION_PIPE_TF32X3;
  return true;
}

bool atc_is(const void* f) {
  return f == atc::fn_of(32) || f == atc::fn_of(64) || f == atc::fn_of(128);
}

// ---- conv weight gradient entry points (gemm.cu conv_wgrad routing)
// args: x, dy, dw, N, H, W, C, K, R, S, stride, pad, P, Q, workspace, ws_bytes
static atc::ConvGeo conv_geo(const uint64_t* a) {
  atc::ConvGeo c;
  c.N = (int)a[3]; c.H = (int)a[4]; c.W = (int)a[5]; c.C = (int)a[6]; c.K = (int)a[7]; c.R = (int)a[8]; c.S = (int)a[9];
  c.stride = (int)a[10]; c.pad = (int)a[11]; c.P = (int)a[12]; c.Q = (int)a[13];
  return c;
}

uint64_t atc_conv_ws_bytes(uint64_t N, uint64_t H, uint64_t W, uint64_t C, uint64_t K, uint64_t R, uint64_t S, uint64_t stride,
                           uint64_t pad) {
  atc::ConvGeo c{(int)N, (int)H, (int)W, (int)C, (int)K, (int)R, (int)S, (int)stride, (int)pad,
                 (int)((H + 2 * pad - R) / stride + 1), (int)((W + 2 * pad - S) / stride + 1)};
  if (C % 32 || K % 4) return 0;
  return atc::ws_bytes(atc::plan_conv(c));
}

bool atc_conv_try_geom(const uint64_t* a, LaunchGeom* g) {
  const atc::ConvGeo c = conv_geo(a);
  if (c.C % 32 || c.K % 4 || c.stride < 1 || c.stride > 8 || c.P <= 0 || c.Q <= 0) return false;
  {
    int QB, PB, npb, nqb;
    atc::conv_blocks(c, QB, PB, npb, nqb);
    if (QB * c.stride > 256 || PB * c.stride > 256) return false;   // TMA box dimension limit
  }
  if (!tmah::al16((const void*)a[0]) || !tmah::al16((const void*)a[1]) || tmah::encoder() == nullptr) return false;
  if ((long long)c.N * c.H * c.W * c.C >= (1LL << 40)) return false;
  atc::Plan pl = atc::plan_conv(c);
  if (pl.split > 1 && (a[14] == 0 || a[15] < atc::ws_bytes(pl))) return false;
  if (!atc::prepare_of(pl.bn, true)) return false;
  g->grid = dim3((unsigned)pl.tiles, (unsigned)pl.split);
  g->block = dim3(atc::NTHR);
  g->smem = atc::smem_of(pl.bn);
  g->func = atc::fn_of(pl.bn, true);
  g->pipe = ORION_PIPE_TF32X3;
  g->sig_ctas = pl.split > 1 ? atc::combine_ctas(pl) : 0;
  return true;
}

bool atc_conv_is(const void* f) {
  return f == atc::fn_of(32, true) || f == atc::fn_of(64, true) || f == atc::fn_of(128, true);
}

int atc_conv_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  const atc::ConvGeo c = conv_geo(a);
  atc::Plan pl = atc::plan_conv(c);
  atc::Params p;
  int QB, PB, npb, nqb;
  atc::conv_blocks(c, QB, PB, npb, nqb);
  const long long RSC = (long long)c.R * c.S * c.C;
  p.trans = pl.trans;
  p.DM = (int)(pl.trans ? RSC : c.K); p.DN = (int)(pl.trans ? c.K : RSC);
  p.K = (int)((long long)c.N * npb * nqb * atc::BK);
  p.C = (float*)a[2]; p.ldc = RSC;
  p.tiles_n = pl.tiles_n; p.tiles = pl.tiles; p.split = pl.split; p.kps = pl.kps;
  p.part = pl.split > 1 ? reinterpret_cast<float*>((unsigned char*)a[14] + WS_TICKET_BYTES) : nullptr;
  p.C = (float*)a[2];
  p.cv_C = c.C; p.cv_S = c.S; p.stride = c.stride; p.pad = c.pad; p.QB = QB; p.PB = PB; p.npb = npb; p.nqb = nqb;
  CUtensorMap mx, mdy;
  const long long dx_dims[4] = {c.C, c.W, c.H, c.N}, dy_dims[4] = {c.K, c.Q, c.P, c.N};
  const int box[4] = {32, QB, PB, 1};
  // with traversal strides the box spans stride x as many x elements (TMA loads ceil(box / stride)
  // of them per dimension), so the x box covers QB * stride columns and PB * stride rows
  const int xbox[4] = {32, QB * c.stride, PB * c.stride, 1};
  if (!tmah::map4d_f32(&mx, (const float*)a[0], dx_dims, xbox, c.stride, c.stride, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)) return ORION_E_CUDA;
  if (!tmah::map4d_f32(&mdy, (const float*)a[1], dy_dims, box, 1, 1, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)) return ORION_E_CUDA;
  // M side: x when trans (M = R*S*C), else dy (M = K)
  return pl.trans ? atc::launch_pair<true>(g, pl, mx, mdy, p, sig, s) : atc::launch_pair<true>(g, pl, mdy, mx, p, sig, s);
}

int atc_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  const long long M = a[4], N = a[5], K = a[6], lda = a[7], ldb = a[8], ldc = a[9];
  atc::Plan pl = atc::plan(M, N, K);
  atc::Params p;
  p.trans = pl.trans;
  p.DM = (int)(pl.trans ? N : M); p.DN = (int)(pl.trans ? M : N); p.K = (int)K;
  p.C = (float*)a[2]; p.ldc = ldc;
  p.tiles_n = pl.tiles_n; p.tiles = pl.tiles; p.split = pl.split; p.kps = pl.kps;
  p.part = nullptr;
  if (pl.split > 1) {
    unsigned char* ws = (unsigned char*)a[11];
    const uint64_t V = (uint64_t)atc::BM * pl.bn;
    (void)V;
    p.part = reinterpret_cast<float*>(ws + WS_TICKET_BYTES);
  }
  const float* Ap = pl.trans ? (const float*)a[1] : (const float*)a[0];   // M side
  const float* Bp = pl.trans ? (const float*)a[0] : (const float*)a[1];   // N side
  const long long ldA = pl.trans ? ldb : lda, ldB = pl.trans ? lda : ldb;
  CUtensorMap mA, mB;
  if (!tmah::map2d_f32_sw(&mA, Ap, K, p.DM, ldA, 32, atc::BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)) return ORION_E_CUDA;
  if (!tmah::map2d_f32_sw(&mB, Bp, K, p.DN, ldB, 32, atc::BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)) return ORION_E_CUDA;
  return atc::launch_pair<false>(g, pl, mA, mB, p, sig, s);
}
