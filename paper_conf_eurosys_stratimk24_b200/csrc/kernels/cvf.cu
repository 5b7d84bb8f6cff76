// Forward convolution as an implicit GEMM on tcgen05 with TMA-built im2col tiles (conv_fwd with
// C % 4 == 0, and the dense B^T GEMM of 1x1 convolutions / Linear layers: gemm flags = 2).
//
// y[n][p][q][k] = sum_{r,s,c} x[n][p*st+r-pad][q*st+s-pad][c] w[k][r][s][c]   (the
// convolutions of the HP ResNet inference and the BE ResNet training step), fp32 through 3xTF32
// (x = hi + lo, D += lo.hi + hi.lo + hi.hi, hi = raw fp32 read as tf32).
//
//  * GEMM rows = a block of output positions (whole output rows: QB = Q columns x PB rows x NB
//    images, <= 128), GEMM K = (tap, 32-channel block) "slabs". A slab of A is ONE 4-D TMA box of the
//    NHWC activations at the tap's shifted origin with traversal strides (stride, stride): TMA
//    builds the im2col tile itself, zero fill = padding, 128-byte swizzle = the UMMA K-major
//    SWIZZLE_128B layout. A slab of B is one box of the [K][R*S][C] weights. No thread computes an
//    address per element.
//  * warps 4-7 form lo = x - trunc_tf32(x) of both operands (elementwise, layout-preserving); warp 8
//    lane 0 issues TMA; warp 9 lane 0 issues the MMAs into three TMEM accumulators (hi*hi of even
//    and of odd slabs, corrections).
//  * small problems (HP inference: a few dozen tiles) split the slabs over a thread-block cluster of
//    <= 8 CTAs along z; the partial tiles meet in distributed shared memory and each CTA sums a
//    row slice of all of them in rank order, so the result is deterministic, needs no workspace and
//    no second launch, and a CTA never waits for a CTA that might not be resident (a cluster is
//    co-scheduled by construction).
//  * one tile per CTA: a CTA lives for a few microseconds, so an HP kernel finds free SMs quickly
//    (kernels are not preemptible).
#include <algorithm>
#include <atomic>
#include <cstdlib>

#include "common.cuh"
#include "tma.cuh"

namespace {
namespace cvf {
using namespace tmah;

constexpr int BM = 128, BK = 32, NTHR = 320, NCONV = 128, TMA_WARP = 8, MMA_WARP = 9, MAX_SPLIT = 8;

template <int BN_>
struct Cfg {
  static constexpr int BN = BN_;
  static constexpr int A_BYTES = BM * BK * 4, B_BYTES = BN * BK * 4;
  static constexpr int STAGE = 2 * (A_BYTES + B_BYTES);   // [A raw][A lo][B raw][B lo]
  static constexpr int STAGES = (196 * 1024) / STAGE > 6 ? 6 : (196 * 1024) / STAGE;
  static constexpr int TS = BN + 4;                       // staging row stride (floats), conflict-free
  static constexpr int SMEM = STAGES * STAGE + 1024 + 256;
  // accumulators: hi*hi of even slabs, of odd slabs, and the correction products (3 BN columns): the
  // tensor core's fp32 accumulation truncates, so shorter chains keep the bias down
  static constexpr int TMEM_COLS = 3 * BN <= 256 ? 256 : 512;
  // kind::tf32: D fp32 (bit 4), A, B tf32 (bits 7, 10), both K-major, N>>3 at 17, M>>4 at 24
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
  static constexpr uint32_t IDESC_BT = IDESC | (1u << 16);   // B MN-major (transposed)
  static_assert(BM * TS * 4 <= STAGES * STAGE, "staging tile fits in the stage ring");
};

struct Params {
  int QB, PB, NB, rows;       // tile = QB x PB x NB output positions (rows <= 128 valid)
  int Q, P, NI;               // output width, height, images (GEMM: Q = M rows, P = NI = 1)
  int nqb, npb;               // position blocks along q and p
  int stride, pad, S, CB;     // conv stride / padding, taps per filter row, 32-channel blocks
  int taps;                   // R * S (1: B is a 2-D map)
  int Kout, tiles_n, nk, kps, split;
  float* y;
  long long ldy;
  const float* bias;
  int dbg;   // measurement switches (ORION_CVF_DEBUG): 1 converters idle, 2 no MMAs, 4 no TMA loads, 8 no epilogue
};

// UMMA descriptor, K-major SWIZZLE_128B: 8-row atoms of 128-byte rows, SBO = 1024 B, layout type 2
__device__ __forceinline__ uint64_t sdesc128(uint32_t addr) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | (1ull << 16) | ((uint64_t)(1024 >> 4) << 32) | (1ull << 46) | (2ull << 61);
}
// UMMA descriptor, MN-major tf32 (B given [K][N]): SWIZZLE_128B with 32-byte atoms (layout type 1,
// TMA CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B), 4-row k-groups 512 B apart, 32-column MN atoms one
// 32 x 32 box (4 KB) apart; k-step j = rows 8j..8j+7 = start + 1024 j
__device__ __forceinline__ uint64_t sdesc_mn(uint32_t addr) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)(4096 >> 4) << 16) | ((uint64_t)(512 >> 4) << 32) | (1ull << 46) | (1ull << 61);
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
__device__ __forceinline__ float4 lo4(const float4 v) {
  return make_float4(v.x - trunc_tf32(v.x), v.y - trunc_tf32(v.y), v.z - trunc_tf32(v.z), v.w - trunc_tf32(v.w));
}
__device__ __forceinline__ void tma_load3d(uint32_t dst, const CUtensorMap* tm, int c0, int c1, int c2, uint32_t bar) {
  asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(dst),
               "l"(tm), "r"(c0), "r"(c1), "r"(c2), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ float4 ld_dsmem4(uint32_t local, uint32_t rank) {
  uint32_t remote;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(local), "r"(rank));
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(remote) : "memory");
  return v;
}

template <int BN, bool BMN>
__global__ void __launch_bounds__(NTHR, 1) cvf_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                                                     Params p, OrionSig sig) {
  using C_ = Cfg<BN>;
  constexpr int A_BYTES = C_::A_BYTES, B_BYTES = C_::B_BYTES, STAGE = C_::STAGE, S = C_::STAGES, TS = C_::TS;
  extern __shared__ __align__(1024) unsigned char cvf_raw[];
  unsigned char* smem = cvf_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(cvf_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * STAGE);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 * S + 2);
  const uint32_t full0 = smem_u32(bars), conv0 = full0 + 8 * S, empty0 = conv0 + 8 * S, done_bar = empty0 + 8 * S;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int z = p.split > 1 ? (int)cluster_rank() : 0;
  const int tile = blockIdx.x;
  const int kb = tile % p.tiles_n, mt = tile / p.tiles_n;
  const int qb = mt % p.nqb, t2 = mt / p.nqb, pb = t2 % p.npb, nb = t2 / p.npb;
  const int q0 = qb * p.QB, p0 = pb * p.PB, n0 = nb * p.NB, k0 = kb * BN;
  const int s0 = z * p.kps, nsl = min(p.nk, s0 + p.kps) - s0;
  const uint32_t tx = (uint32_t)(p.QB * p.PB * p.NB * 128 + BN * 128);
  // no K split: the epilogue writes rows straight from TMEM (one 128-byte run per thread per
  // 32-column chunk), skipping the staging tile and the reduction pass
  const bool direct = p.split == 1;
  const bool dvec = (p.ldy & 3) == 0 && (reinterpret_cast<uintptr_t>(p.y) & 15) == 0;

  if (tid == 0) {
    for (int s = 0; s < S; s++) { mbar_init(full0 + 8 * s, 1); mbar_init(conv0 + 8 * s, NCONV / 32); mbar_init(empty0 + 8 * s, 1); }
    mbar_init(done_bar, 1);
    fence_barrier_init();
  }
  if (warp == TMA_WARP && lane == 0) { prefetch_tmap(&tmA); prefetch_tmap(&tmB); }
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(C_::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp == TMA_WARP) {
    if (lane == 0) {
      int tap = s0 / p.CB, cb = s0 - tap * p.CB, r = tap / p.S, sx = tap - r * p.S;   // slab s0
#pragma unroll 1
      for (int it = 0; it < nsl; it++) {
        const int s = it % S;
        if (it >= S) mbar_wait(empty0 + 8 * s, ((uint32_t)(it / S) & 1u) ^ 1u);
        const uint32_t st = smem_u32(smem + s * STAGE), bar = full0 + 8 * s;
        if (p.dbg & 4) { mbar_arrive(bar); continue; }   // (counters unused in this measurement mode)
        mbar_expect(bar, tx);
        tma_load4d(st, &tmA, cb * 32, q0 * p.stride + sx - p.pad, p0 * p.stride + r - p.pad, n0, bar);
        if (BMN) {   // B [K][N]: BN / 32 MN-major boxes of 32 k-rows
#pragma unroll
          for (int j = 0; j < BN / 32; j++) tma_load2d(st + 2 * A_BYTES + 4096 * j, &tmB, k0 + 32 * j, cb * 32, bar);
        } else if (p.taps == 1) tma_load2d(st + 2 * A_BYTES, &tmB, cb * 32, k0, bar);
        else tma_load3d(st + 2 * A_BYTES, &tmB, cb * 32, tap, k0, bar);
        if (++cb == p.CB) { cb = 0; ++tap; if (++sx == p.S) { sx = 0; ++r; } }   // next slab, no divisions
      }
    }
  } else if (warp >= 4 && warp < TMA_WARP) {
    // lo = x - trunc_tf32(x) of the loaded rows of A (garbage rows >= p.rows only feed discarded
    // accumulator rows) and of B
    const int ct = tid - 128;
    const int aq = p.rows * (BK / 4);
#pragma unroll 1
    for (int it = 0; it < nsl; it++) {
      const int s = it % S;
      mbar_wait(full0 + 8 * s, (uint32_t)(it / S) & 1u);
      unsigned char* st = smem + s * STAGE;
      const float4* ahi = reinterpret_cast<const float4*>(st);
      float4* alo = reinterpret_cast<float4*>(st + A_BYTES);
      const float4* bhi = reinterpret_cast<const float4*>(st + 2 * A_BYTES);
      float4* blo = reinterpret_cast<float4*>(st + 2 * A_BYTES + B_BYTES);
      if (p.dbg & 1) {
        __syncwarp();
        if (lane == 0) mbar_arrive(conv0 + 8 * s);
        continue;
      }
      float4 va[8], vb[BN / 16];
#pragma unroll
      for (int j = 0; j < 8; j++) {
        const int i = ct + NCONV * j;
        if (i < aq) va[j] = ahi[i];
      }
#pragma unroll
      for (int j = 0; j < BN / 16; j++) vb[j] = bhi[ct + NCONV * j];
#pragma unroll
      for (int j = 0; j < 8; j++) {
        const int i = ct + NCONV * j;
        if (i < aq) alo[i] = lo4(va[j]);
      }
#pragma unroll
      for (int j = 0; j < BN / 16; j++) blo[ct + NCONV * j] = lo4(vb[j]);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(conv0 + 8 * s);
    }
  } else if (warp == MMA_WARP && lane == 0) {
#pragma unroll 1
    for (int it = 0; it < nsl; it++) {
      const int s = it % S;
      const uint32_t ph = (uint32_t)(it / S) & 1u;
      mbar_wait(full0 + 8 * s, ph);
      mbar_wait(conv0 + 8 * s, ph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t st = smem_u32(smem + s * STAGE);
      const uint32_t a_hi = st, a_lo = st + A_BYTES, b_hi = st + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
      const uint32_t d_main = tmem + (uint32_t)((it & 1) * BN), d_corr = tmem + 2 * BN;
#pragma unroll
      for (int j = 0; j < ((p.dbg & 2) ? 0 : BK / 8); j++) {
        const uint64_t dah = sdesc128(a_hi + 32 * j), dal = sdesc128(a_lo + 32 * j);
        const uint64_t dbh = BMN ? sdesc_mn(b_hi + 1024 * j) : sdesc128(b_hi + 32 * j);
        const uint64_t dbl = BMN ? sdesc_mn(b_lo + 1024 * j) : sdesc128(b_lo + 32 * j);
        constexpr uint32_t ID = BMN ? C_::IDESC_BT : C_::IDESC;
        mma_tf32(d_corr, dal, dbh, ID, (it | j) != 0);
        mma_tf32(d_corr, dah, dbl, ID, 1);
        mma_tf32(d_main, dah, dbh, ID, ((it >> 1) | j) != 0);
      }
      mma_commit(empty0 + 8 * s);
    }
    mma_commit(done_bar);
  } else if (warp < 4 && !(p.dbg & 8)) {
    // TMEM -> registers -> staging tile [128][TS] (the stage ring is idle once done_bar fired)
    mbar_wait(done_bar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    float* tilep = reinterpret_cast<float*>(smem);
    float* drow = nullptr;   // direct mode: this thread's (tile row = TMEM lane) output row
    if (direct && tid < p.rows) {
      const int q = tid % p.QB, t = tid / p.QB, pp = t % p.PB, nn = t / p.PB;
      const int qa = q0 + q, pa = p0 + pp, na = n0 + nn;
      if (qa < p.Q && pa < p.P && na < p.NI) drow = p.y + ((long long)(na * p.P + pa) * p.Q + qa) * p.ldy;
    }
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t ev[32], ov[32], cv[32];
      const uint32_t base = tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)c0;
      tmem_ld32(base, ev);
      tmem_ld32(base + 2 * BN, cv);
      if (nsl > 1) tmem_ld32(base + BN, ov);
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (nsl <= 1) {
#pragma unroll
        for (int j = 0; j < 32; j++) ov[j] = 0u;   // +0.0f: the odd chain is empty
      }
      if (direct) {   // no split: this thread's output row straight from registers (+ bias)
        if (drow) {
#pragma unroll
          for (int j = 0; j < 32; j += 4) {
            const int n = k0 + c0 + j;
            float t[4];
#pragma unroll
            for (int i = 0; i < 4; i++)
              t[i] = ((__uint_as_float(ev[j + i]) + __uint_as_float(ov[j + i])) + __uint_as_float(cv[j + i])) +
                     (p.bias && n + i < p.Kout ? __ldg(p.bias + n + i) : 0.f);
            if (dvec && n + 3 < p.Kout) *reinterpret_cast<float4*>(drow + n) = make_float4(t[0], t[1], t[2], t[3]);
            else
              for (int i = 0; i < 4 && n + i < p.Kout; i++) drow[n + i] = t[i];
          }
        }
        continue;
      }
#pragma unroll
      for (int j = 0; j < 32; j += 4) {
        float4 v;
        v.x = (__uint_as_float(ev[j]) + __uint_as_float(ov[j])) + __uint_as_float(cv[j]);
        v.y = (__uint_as_float(ev[j + 1]) + __uint_as_float(ov[j + 1])) + __uint_as_float(cv[j + 1]);
        v.z = (__uint_as_float(ev[j + 2]) + __uint_as_float(ov[j + 2])) + __uint_as_float(cv[j + 2]);
        v.w = (__uint_as_float(ev[j + 3]) + __uint_as_float(ov[j + 3])) + __uint_as_float(cv[j + 3]);
        *reinterpret_cast<float4*>(tilep + tid * TS + c0 + j) = v;
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (p.split > 1) cluster_sync();   // every partial tile of the cluster is staged

  // ---------------- sum the partial tiles of this CTA's row slice in rank order, store
  if (!(p.dbg & 8) && !direct) {
    const int per = (p.rows + p.split - 1) / p.split;
    const int r_lo = z * per, r_hi = min(p.rows, r_lo + per);
    constexpr int QPR = BN / 4;
    const uint32_t tbase = smem_u32(smem);
    const float* tilep = reinterpret_cast<const float*>(smem);
    const bool vec = (p.ldy & 3) == 0 && (reinterpret_cast<uintptr_t>(p.y) & 15) == 0;
#pragma unroll 1
    for (int e = tid; e < (r_hi - r_lo) * QPR; e += NTHR) {
      const int r = r_lo + e / QPR, c = (e % QPR) * 4;
      const int n = k0 + c;
      if (n >= p.Kout) continue;
      const int q = r % p.QB, t = r / p.QB, pp = t % p.PB, nn = t / p.PB;
      const int qa = q0 + q, pa = p0 + pp, na = n0 + nn;
      if (qa >= p.Q || pa >= p.P || na >= p.NI) continue;
      float4 v;
      if (p.split == 1) {
        v = *reinterpret_cast<const float4*>(tilep + r * TS + c);
      } else {
        // all remote loads in flight at once (one DSMEM latency, not split of them), then the
        // fixed rank-order sum
        const uint32_t off = tbase + (uint32_t)((r * TS + c) * 4);
        float4 w[MAX_SPLIT];
#pragma unroll
        for (int zz = 0; zz < MAX_SPLIT; zz++)
          if (zz < p.split) w[zz] = ld_dsmem4(off, (uint32_t)zz);
        v = w[0];
#pragma unroll
        for (int zz = 1; zz < MAX_SPLIT; zz++)
          if (zz < p.split) { v.x += w[zz].x; v.y += w[zz].y; v.z += w[zz].z; v.w += w[zz].w; }
      }
      float* dst = p.y + ((long long)(na * p.P + pa) * p.Q + qa) * p.ldy + n;
      if (p.bias) {
        if (n < p.Kout) v.x += __ldg(p.bias + n);
        if (n + 1 < p.Kout) v.y += __ldg(p.bias + n + 1);
        if (n + 2 < p.Kout) v.z += __ldg(p.bias + n + 2);
        if (n + 3 < p.Kout) v.w += __ldg(p.bias + n + 3);
      }
      if (vec && n + 3 < p.Kout) {
        *reinterpret_cast<float4*>(dst) = v;
      } else {
        const float tv[4] = {v.x, v.y, v.z, v.w};
        for (int i = 0; i < 4 && n + i < p.Kout; i++) dst[i] = tv[i];
      }
    }
  }
  if (p.split > 1) cluster_sync();   // peers are done reading this CTA's tile
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C_::TMEM_COLS) : "memory");
  }
  orion_signal(sig);
}

// ---------------------------------------------------------------- host side
struct Shape {   // one forward convolution (or B^T GEMM as a 1x1 convolution over Q = M positions)
  const float* x; const float* w; float* y; const float* bias;
  long long NI, H, W, C, K, R, S, stride, pad, P, Q;
  long long ldx, ldw, ldy;   // GEMM strides (conv: C, R*S*C, K)
  bool gemm;
  bool bmn;                  // GEMM with B given [K][N] (flags = 0), not [N][K]
};
struct Plan { int BN, QB, PB, NB, nqb, npb, nnb, tiles, tiles_n, nk, kps, split; };

inline long long cdivl(long long a, long long b) { return (a + b - 1) / b; }

inline bool shape_ok(const Shape& s) {
  if (s.C < 4 || s.C % 4 || s.K < 4 || s.NI <= 0 || s.P <= 0 || s.Q <= 0) return false;
  if (s.R * s.S > 65535 || s.stride < 1 || s.stride > 2 || s.pad < 0) return false;   // box extent QB*stride <= 256
  if (!al16(s.x) || !al16(s.w) || (s.ldx % 4) || (s.ldw % 4)) return false;
  if (s.NI * s.P * s.Q >= (1LL << 31) || s.K >= (1LL << 31)) return false;
  return encoder() != nullptr;
}

template <int BN, bool BMN = false>
bool prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  const bool okk = cudaFuncSetAttribute((const void*)cvf_kernel<BN, BMN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::SMEM) == cudaSuccess;
  if (okk) done.store(1, std::memory_order_release);
  return okk;
}

// clusters of `split` CTAs the device runs at once (cudaOccupancyMaxActiveClusters; measured once per
// (BN, split)): GPC sizes, not the SM count, bound a cluster wave (e.g. 15 clusters of 8 on 148 SMs)
inline int max_clusters(int BN, int split) {
  static std::atomic<int> cache[2][MAX_SPLIT + 1];
  const int b = BN == 128 ? 1 : 0;
  int v = cache[b][split].load(std::memory_order_relaxed);
  if (v > 0) return v;
  int n = 0;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(1, 1, (unsigned)split); cfg.blockDim = dim3(NTHR);
  cfg.dynamicSmemBytes = BN == 128 ? Cfg<128>::SMEM : Cfg<64>::SMEM;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 1; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = (unsigned)split;
  cfg.attrs = at; cfg.numAttrs = 1;
  const bool ok = BN == 128 ? prepare<128>() && cudaOccupancyMaxActiveClusters(&n, cvf_kernel<128, false>, &cfg) == cudaSuccess
                            : prepare<64>() && cudaOccupancyMaxActiveClusters(&n, cvf_kernel<64, false>, &cfg) == cudaSuccess;
  if (!ok || n <= 0) { (void)cudaGetLastError(); n = 148 / split; }
  cache[b][split].store(n, std::memory_order_relaxed);
  return n;
}

inline Plan plan(const Shape& s) {
  Plan pl;
  if (s.Q <= 128) {
    pl.QB = (int)s.Q;
    const long long pbmax = std::min<long long>(s.P, 128 / s.Q);
    pl.npb = (int)cdivl(s.P, pbmax);
    pl.PB = (int)cdivl(s.P, pl.npb);                      // balanced row blocks
    pl.NB = pl.PB == s.P ? (int)std::max<long long>(1, std::min<long long>(s.NI, 128 / (s.P * s.Q))) : 1;
    if (pl.NB > 1) pl.NB = (int)cdivl(s.NI, cdivl(s.NI, pl.NB));
  } else {
    pl.QB = 128; pl.PB = 1; pl.NB = 1; pl.npb = (int)s.P;
  }
  pl.nqb = (int)cdivl(s.Q, pl.QB);
  pl.nnb = (int)cdivl(s.NI, pl.NB);
  const long long tiles_m = (long long)pl.nqb * pl.npb * pl.nnb;
  static const int force_bn = getenv("ORION_CVF_BN") ? atoi(getenv("ORION_CVF_BN")) : 0;   // tuning knobs
  static const int max_split = getenv("ORION_CVF_MAXSPLIT") ? std::max(1, std::min(MAX_SPLIT, atoi(getenv("ORION_CVF_MAXSPLIT")))) : MAX_SPLIT;
  // BN = 128 whenever the layer has 128+ output channels: one N=128 MMA costs little more than an
  // N=64 one (measured sweep over the HP ResNet-50 shapes, tools/bench_kernels.py conv)
  pl.BN = force_bn == 64 || force_bn == 128 ? force_bn : s.K >= 128 ? 128 : 64;
  pl.tiles_n = (int)cdivl(s.K, pl.BN);
  pl.tiles = (int)(tiles_m * pl.tiles_n);
  pl.nk = (int)(s.R * s.S * cdivl(s.C, 32));
  int split = 1;
  if (pl.tiles < 148) split = std::max(1, std::min({max_split, 148 / pl.tiles, pl.nk / 2}));
  // a cluster of `split` CTAs needs `split` free SMs in one GPC: keep all clusters in one wave
  while (split > 1 && pl.tiles > max_clusters(pl.BN, split)) split--;
  pl.kps = (int)cdivl(pl.nk, split);
  pl.split = (int)cdivl(pl.nk, pl.kps);
  return pl;
}


inline bool geom(const Shape& s, LaunchGeom* g) {
  if (!shape_ok(s)) return false;
  const Plan pl = plan(s);
  const bool okp = s.bmn ? (pl.BN == 128 ? prepare<128, true>() : prepare<64, true>()) : (pl.BN == 128 ? prepare<128>() : prepare<64>());
  if (!okp) return false;
  g->grid = dim3((unsigned)pl.tiles, 1, (unsigned)pl.split);
  g->block = dim3(NTHR);
  g->smem = pl.BN == 128 ? Cfg<128>::SMEM : Cfg<64>::SMEM;
  g->func = s.bmn ? (pl.BN == 128 ? (const void*)cvf_kernel<128, true> : (const void*)cvf_kernel<64, true>)
                  : (pl.BN == 128 ? (const void*)cvf_kernel<128, false> : (const void*)cvf_kernel<64, false>);
  g->pipe = ORION_PIPE_TF32X3;
  return true;
}

inline bool is(const void* f) {
  return f == (const void*)cvf_kernel<128, false> || f == (const void*)cvf_kernel<64, false> || f == (const void*)cvf_kernel<128, true> ||
         f == (const void*)cvf_kernel<64, true>;
}

template <int BN, bool BMN>
int launch_t(const Shape& s, const Plan& pl, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  if (!prepare<BN, BMN>()) return ORION_E_CUDA;
  CUtensorMap ma, mb;
  // activations: {C, W, H, N} (GEMM: {K, M, 1, 1}); box {32, QB*stride, PB*stride, NB}, traversal strides
  // (stride, stride): TMA gathers QB x PB x NB positions of one tap (ceil(box / stride) per dim)
  const long long dims[4] = {s.C, s.gemm ? s.Q : s.W, s.gemm ? 1 : s.H, s.gemm ? 1 : s.NI};
  const int box[4] = {32, (int)(pl.QB * s.stride), (int)(pl.PB * s.stride), pl.NB};
  {
    encode_fn e = encoder();
    cuuint64_t gd[4] = {(cuuint64_t)dims[0], (cuuint64_t)dims[1], (cuuint64_t)dims[2], (cuuint64_t)dims[3]};
    cuuint64_t gs[3] = {(cuuint64_t)s.ldx * 4, (cuuint64_t)s.ldx * dims[1] * 4, (cuuint64_t)s.ldx * dims[1] * dims[2] * 4};
    cuuint32_t bx[4] = {(cuuint32_t)box[0], (cuuint32_t)box[1], (cuuint32_t)box[2], (cuuint32_t)box[3]};
    cuuint32_t es[4] = {1, (cuuint32_t)s.stride, (cuuint32_t)s.stride, 1};
    if (e(&ma, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, (void*)s.x, gd, gs, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
          CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return ORION_E_CUDA;
  }
  if (BMN) {   // B [C (reduction)][K (outputs)] row-major: 32 x 32 MN-major boxes
    if (!map2d_f32_sw(&mb, s.w, s.C, s.K, s.ldw, 32, 32, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)) return ORION_E_CUDA;
  } else if (s.R * s.S == 1) {
    if (!map2d_f32_sw(&mb, s.w, s.K, s.C, s.ldw, 32, BN, CU_TENSOR_MAP_SWIZZLE_128B)) return ORION_E_CUDA;
  } else {
    encode_fn e = encoder();
    cuuint64_t gd[3] = {(cuuint64_t)s.C, (cuuint64_t)(s.R * s.S), (cuuint64_t)s.K};
    cuuint64_t gs[2] = {(cuuint64_t)s.C * 4, (cuuint64_t)s.ldw * 4};
    cuuint32_t bx[3] = {32, 1, (cuuint32_t)BN};
    cuuint32_t es[3] = {1, 1, 1};
    if (e(&mb, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, (void*)s.w, gd, gs, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
          CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return ORION_E_CUDA;
  }
  Params p;
  p.QB = pl.QB; p.PB = pl.PB; p.NB = pl.NB; p.rows = pl.QB * pl.PB * pl.NB;
  p.Q = (int)s.Q; p.P = (int)s.P; p.NI = (int)s.NI; p.nqb = pl.nqb; p.npb = pl.npb;
  p.stride = (int)s.stride; p.pad = (int)s.pad; p.S = (int)s.S; p.CB = (int)cdivl(s.C, 32); p.taps = (int)(s.R * s.S);
  p.Kout = (int)s.K; p.tiles_n = pl.tiles_n; p.nk = pl.nk; p.kps = pl.kps; p.split = pl.split;
  p.y = s.y; p.ldy = s.ldy; p.bias = s.bias;
  static const int dbg = getenv("ORION_CVF_DEBUG") ? atoi(getenv("ORION_CVF_DEBUG")) : 0;
  p.dbg = dbg;
  if (pl.split == 1) {
    cvf_kernel<BN, BMN><<<g.grid, g.block, g.smem, st>>>(ma, mb, p, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = g.grid; cfg.blockDim = g.block; cfg.dynamicSmemBytes = g.smem; cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 1; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = (unsigned)pl.split;
  cfg.attrs = at; cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, cvf_kernel<BN, BMN>, ma, mb, p, sig) == cudaSuccess ? 0 : ORION_E_CUDA;
}

inline int launch(const Shape& s, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  const Plan pl = plan(s);
  if (s.bmn) return pl.BN == 128 ? launch_t<128, true>(s, pl, g, sig, st) : launch_t<64, true>(s, pl, g, sig, st);
  return pl.BN == 128 ? launch_t<128, false>(s, pl, g, sig, st) : launch_t<64, false>(s, pl, g, sig, st);
}

// conv_fwd args: x, w, y, N, H, W, C, K, R, S, stride, pad, P, Q, workspace, ws_bytes
inline Shape conv_shape(const uint64_t* a) {
  Shape s;
  s.x = (const float*)a[0]; s.w = (const float*)a[1]; s.y = (float*)a[2]; s.bias = nullptr;
  s.NI = (long long)a[3]; s.H = (long long)a[4]; s.W = (long long)a[5]; s.C = (long long)a[6]; s.K = (long long)a[7];
  s.R = (long long)a[8]; s.S = (long long)a[9]; s.stride = (long long)a[10]; s.pad = (long long)a[11];
  s.P = (long long)a[12]; s.Q = (long long)a[13];
  s.ldx = s.C; s.ldw = s.R * s.S * s.C; s.ldy = s.K; s.gemm = false; s.bmn = false;
  if (s.R == 1 && s.S == 1 && s.stride == 1 && s.pad == 0) {   // pointwise: one GEMM over all positions
    s.gemm = true; s.Q = s.NI * s.P * s.Q; s.P = 1; s.NI = 1; s.H = 1; s.W = s.Q;
  }
  return s;
}
// gemm args (flags = 2: B^T [N][ldb]; flags = 0: B [K][ldb]): A [M][lda], C [M][ldc], bias
inline Shape gemm_shape(const uint64_t* a) {
  Shape s;
  s.x = (const float*)a[0]; s.w = (const float*)a[1]; s.y = (float*)a[2]; s.bias = (const float*)a[3];
  s.Q = (long long)a[4]; s.K = (long long)a[5]; s.C = (long long)a[6];
  s.NI = 1; s.P = 1; s.H = 1; s.W = s.Q; s.R = 1; s.S = 1; s.stride = 1; s.pad = 0;
  s.ldx = (long long)a[7]; s.ldw = (long long)a[8]; s.ldy = (long long)a[9]; s.gemm = true; s.bmn = (int)a[10] == 0;
  return s;
}

}  // namespace cvf
}  // namespace

bool cvf_conv_try_geom(const uint64_t* a, LaunchGeom* g) {
  static const bool off = getenv("ORION_CVF_OFF") != nullptr;   // A/B switch for measurements
  return !off && cvf::geom(cvf::conv_shape(a), g);
}
bool cvf_gemm_try_geom(const uint64_t* a, LaunchGeom* g) {
  static const bool off = getenv("ORION_CVF_OFF") != nullptr;
  if (off || ((int)a[10] != 2 && (int)a[10] != 0)) return false;
  return cvf::geom(cvf::gemm_shape(a), g);
}
bool cvf_is(const void* f) { return cvf::is(f); }
int cvf_conv_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) { return cvf::launch(cvf::conv_shape(a), g, sig, s); }
int cvf_gemm_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) { return cvf::launch(cvf::gemm_shape(a), g, sig, s); }
