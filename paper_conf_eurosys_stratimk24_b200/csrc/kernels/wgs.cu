// Streaming weight-gradient GEMM (gemm flags = 1): C[M][N] = sum_k A[k][m] B[k][n], i.e.
// dW = dy^T x of a 1x1 convolution or Linear layer summed over K = N*H*W (or batch) rows
// (cuDNN/cuBLAS weight-gradient kernels in the paper's PyTorch runs).
//
// At MobileNetV2's early layers the reduction runs over 1.2 M rows of 16-96 channels: the op reads
// 0.2-0.5 GB once and does ~7-14 flops per byte, so it is HBM-bound on the FFMA pipe (SURVEY
// §8(d)). Design (sm_100a):
//  * one producer thread streams R-row blocks of both operands with 2-D TMA into a ring of shared
//    memory stages (mbarrier full/empty pairs); zero fill covers ragged tiles;
//  * eight consumer warps are row groups: warp g multiplies rows g, g+8, ... of every stage. The
//    "lane" operand (the wider of dy / x, chosen per shape) gives lane l the columns l, l+32, ..
//    (conflict-free 4-byte shared loads); the other operand's NB values of the row are read as
//    warp-uniform 16-byte broadcasts; each lane keeps an MI x NB register block;
//  * the eight row-group blocks are added in warp order, each CTA writes its fp32 partial tile and
//    the last CTA of every tile sums the K splits in split order in fp64 (combine_splits).
// The tile shape, the K split and the stage size are functions of (M, N, K) only, so results are
// bitwise reproducible and independent of the SM partition the kernel runs in.
#include <cstdlib>

#include "common.cuh"
#include "tma.cuh"

namespace {
namespace wgs {
using namespace tmah;

constexpr int NCW = 8;                    // warps = row groups; lane 0 of warp 0 also issues the TMA loads
constexpr int NTHR = NCW * 32;            // 8 warps: two CTAs (16 warps, 4 per SM sub-partition) at <= 128 registers
constexpr int STAGE_BUDGET = 96 * 1024;   // stage ring per CTA: two CTAs per SM

struct Plan {
  int trans;            // 0: lane operand = A (C[l][q]); 1: lane operand = B (C[q][l])
  int mi, nb;           // register block: MI lane columns x NB broadcast columns
  int tiles_l, tiles_q, split, kps, R, stages;
  int smem;
};

struct Params {
  int DL, DQ, K, trans;
  float* C;
  long long ldc;
  int tiles_l, tiles_q, split, kps, R, stages;
  unsigned int* tickets;
  float* part;     // [tile][split][V] fp32 partial tiles
  double* gpart;   // [tile][groups][V] fp64 group sums (two-level combine)
};

// register blocks with <= 72 accumulators; two CTAs of 256 threads per SM put 4 warps on each
// 16 K-register sub-partition: <= 128 registers per thread
__host__ __device__ constexpr bool blk_ok(int mi, int nb) { return mi * nb <= 72; }
constexpr int MAXREG = 128;

inline int pow2_floor(int v) {
  int p = 1;
  while (p * 2 <= v) p *= 2;
  return p;
}

// stage size (KB) of the ring: a tuning knob (ORION_WGS_STAGE_KB, read once; default 32), never a
// function of the partition, so results stay independent of where the kernel runs
inline int stage_kb() {
  static const int kb = [] {
    const char* e = getenv("ORION_WGS_STAGE_KB");
    const int v = e ? atoi(e) : 32;
    return v >= 4 && v <= 48 ? v : 32;
  }();
  return kb;
}

inline int stage_rows(int rowf) {
  int r = pow2_floor(stage_kb() * 1024 / (rowf * 4));
  return r < 32 ? 32 : (r > 256 ? 256 : r);
}

inline int smem_bytes(int mi, int nb, int R, int stages) {
  const int tl = 32 * mi, V = tl * nb;
  int body = stages * R * (tl + nb) * 4;
  const int red = NCW * V * 4, comb = (V + NTHR) * 8;
  if (red > body) body = red;
  if (comb > body) body = comb;
  return 256 + body;   // barriers, stage / reduction area
}

// Shape-only plan (never the SM count of the partition): pick the operand roles and register
// block by a three-term time model (FFMA issue, HBM bytes, L2 re-reads), then split K so that about
// two CTAs per SM of a 148-SM B200 stream, keeping the partial-tile traffic small.
inline int split_for(long long M, long long N, long long K, int tiles, int R, int mi, int nb) {
  // at most one wave of two CTAs per SM (a 148-SM B200 constant, not the partition's count)
  long long split = tiles >= 296 ? 1 : 296 / tiles;
  const long long kmax = K / (2LL * R);   // >= 2 stages per split
  if (split > kmax) split = kmax > 0 ? kmax : 1;
  // partial tiles (written once, read once) within ~25 % of the operand bytes
  const long long V = 32LL * mi * nb;
  const long long pmax = (4 * K * (M + N)) / (32 * tiles * V);
  if (split > pmax) split = pmax > 0 ? pmax : 1;
  if (split > 1024) split = 1024;
  return (int)split;
}

inline Plan plan(long long M, long long N, long long K) {
  static const int MIS[3] = {1, 2, 3};
  static const int NBS[5] = {8, 16, 24, 32, 4};
  Plan best{};
  double best_cost = 1e300;
  for (int trans = 0; trans < 2; trans++) {
    const long long DL = trans ? N : M, DQ = trans ? M : N;
    for (int mi : MIS)
      for (int nb : NBS) {
        if (!blk_ok(mi, nb)) continue;
        const long long tl = cdiv(DL, 32 * mi), tq = cdiv(DQ, nb), tiles = tl * tq;
        if (tiles > (1 << 20)) continue;
        const int R = stage_rows(32 * mi + nb);
        const long long split = split_for(M, N, K, (int)tiles, R, mi, nb);
        const long long ctas = tiles * split, waves = cdiv(ctas, 296);
        const double eff = (double)ctas / (double)(waves * 296);   // fraction of the CTA slots kept busy
        const double issue = (double)tiles * (mi * nb + mi + nb / 4 + 3);   // warp instructions per row
        const double t_fma = (double)K * issue / (148.0 * 4 * 1.9e9) / eff;
        const double t_hbm = 4.0 * K * (M + N) / 6.5e12 / (eff < 0.5 ? 2 * eff : 1.0);
        const double t_l2 = 4.0 * K * tiles * (32 * mi + nb) / 20e12;
        double cost = t_fma > t_hbm ? t_fma : t_hbm;
        if (t_l2 > cost) cost = t_l2;
        cost += 1e-9 * tiles;   // tie-break towards fewer tiles
        if (cost < best_cost) {
          best_cost = cost;
          best.trans = trans; best.mi = mi; best.nb = nb; best.tiles_l = (int)tl; best.tiles_q = (int)tq;
          best.R = R; best.split = (int)split;
        }
      }
  }
  const int rowf = 32 * best.mi + best.nb;
  best.stages = STAGE_BUDGET / (best.R * rowf * 4);
  if (best.stages > 8) best.stages = 8;
  if (best.stages < 2) best.stages = 2;
  long long kps = cdiv(cdiv(K, best.split), best.R) * best.R;
  best.kps = (int)kps;
  best.split = (int)cdiv(K, kps);
  best.smem = smem_bytes(best.mi, best.nb, best.R, best.stages);
  return best;
}

inline uint64_t ws_bytes(const Plan& p) {
  if (p.split <= 1) return 0;
  const uint64_t tiles = (uint64_t)p.tiles_l * p.tiles_q, V = 32ull * p.mi * p.nb;
  return WS_TICKET_BYTES + tiles * p.split * V * 4 + 16 + tiles * (uint64_t)combine_rows(p.split) * V * 8;
}

template <int MI, int NB>
__global__ void __maxnreg__(MAXREG) wgs_kernel(const __grid_constant__ CUtensorMap tmL, const __grid_constant__ CUtensorMap tmQ,
                                                     Params p, OrionSig sig) {
  constexpr int TL = 32 * MI, ROWF = TL + NB, V = TL * NB;
  // (pointers derived from the shared array itself, so the compiler emits LDS, not generic loads;
  // dynamic shared memory is 128-byte aligned, more than TMA's 16 bytes without swizzle)
  extern __shared__ __align__(128) unsigned char wgs_smem[];
  uint64_t* bars = reinterpret_cast<uint64_t*>(wgs_smem);   // full[stages], empty[stages]
  float* ring = reinterpret_cast<float*>(wgs_smem + 256);
  const int R = p.R, S = p.stages, stage_floats = R * ROWF;
  const uint32_t full0 = smem_u32(bars), empty0 = full0 + 8 * S;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int tile = blockIdx.x, z = blockIdx.y;
  const int l0 = (tile % p.tiles_l) * TL, q0 = (tile / p.tiles_l) * NB;
  const int k0 = z * p.kps, k1 = min(p.K, k0 + p.kps);
  const int nst = (k1 - k0 + R - 1) / R;

  if (tid == 0) {
    for (int s = 0; s < S; s++) { mbar_init(full0 + 8 * s, 1); mbar_init(empty0 + 8 * s, NCW); }
    // (released[] below is zeroed before the first arrival)
    fence_barrier_init();
    prefetch_tmap(&tmL);
    prefetch_tmap(&tmQ);
  }
  __syncthreads();

  // accumulator pairs (columns 2j, 2j+1 of the broadcast operand): packed FFMA2, two FMAs per issue
  // slot (same per-lane rounding as fmaf: results bit-identical to the scalar form)
  float2 acc[MI][NB / 2];
#pragma unroll
  for (int i = 0; i < MI; i++)
#pragma unroll
    for (int j = 0; j < NB / 2; j++) acc[i][j] = make_float2(0.f, 0.f);

  // producer: the slot of stage `it` is refilled with stage it + S by the warp that releases it last
  // (a per-slot arrival count in shared memory), so all S slots are in flight and no warp waits for
  // another to issue loads. Stage `it` lands in slot it % S; its full barrier completes phase
  // (it / S) & 1.
  __shared__ unsigned int released[8];
  if (tid < 8) released[tid] = 0u;
  __syncthreads();
  const uint32_t tx = (uint32_t)stage_floats * 4;
  auto produce = [&](int it) {
    const int s = it % S;
    const uint32_t bar = full0 + 8 * s, dst = smem_u32(ring + (size_t)s * stage_floats);
    mbar_expect(bar, tx);
    tma_load2d(dst, &tmL, l0, k0 + it * R, bar);
    tma_load2d(dst + (uint32_t)(R * TL * 4), &tmQ, q0, k0 + it * R, bar);
  };
  if (tid == 0)
    for (int it = 0; it < S && it < nst; it++) produce(it);
#pragma unroll 1
  for (int it = 0; it < nst; it++) {
    const int s = it % S;
    mbar_wait(full0 + 8 * s, (uint32_t)(it / S) & 1u);
    const float* Ls = ring + (size_t)s * stage_floats + lane;
    const float4* Qs = reinterpret_cast<const float4*>(ring + (size_t)s * stage_floats + R * TL);
    const int rows = min(R, k1 - (k0 + it * R));
    // two rows per trip when the register block leaves room (both rows' loads issued before the
    // first row's FMAs: the LDS latency of one row hides behind the other's arithmetic); the
    // accumulation order is unchanged (row r, then row r + NCW)
    constexpr int RU = MI * NB <= 48 ? 2 : 1;
    auto fma_row = [&](const float (&lv)[MI], const float4 (&qv)[NB / 4]) {
#pragma unroll
      for (int j = 0; j < NB / 4; j++)
#pragma unroll
        for (int i = 0; i < MI; i++) {
          ffma2(acc[i][2 * j], lv[i], make_float2(qv[j].x, qv[j].y));
          ffma2(acc[i][2 * j + 1], lv[i], make_float2(qv[j].z, qv[j].w));
        }
    };
    auto ld_row = [&](int r, float (&lv)[MI], float4 (&qv)[NB / 4]) {
#pragma unroll
      for (int i = 0; i < MI; i++) lv[i] = Ls[r * TL + 32 * i];
#pragma unroll
      for (int j = 0; j < NB / 4; j++) qv[j] = Qs[r * (NB / 4) + j];
    };
    int r = warp;
    if (RU == 2) {
#pragma unroll 1
      for (; r + NCW < rows; r += 2 * NCW) {
        float lv0[MI], lv1[MI];
        float4 q0[NB / 4], q1[NB / 4];
        ld_row(r, lv0, q0);
        ld_row(r + NCW, lv1, q1);
        fma_row(lv0, q0);
        fma_row(lv1, q1);
      }
    }
#pragma unroll 1
    for (; r < rows; r += NCW) {
      float lv[MI];
      float4 qv[NB / 4];
      ld_row(r, lv, qv);
      fma_row(lv, qv);
    }
    __syncwarp();
    if (lane == 0) {
      // this warp is done reading slot s; the last of the NCW warps to get here refills it (the
      // empty barrier orders every warp's reads before the async-proxy TMA write)
      mbar_arrive(empty0 + 8 * s);
      if (atomicAdd(&released[s], 1u) == NCW - 1) {
        released[s] = 0u;
        if (it + S < nst) {
          mbar_wait(empty0 + 8 * s, (uint32_t)(it / S) & 1u);
          produce(it + S);
        }
      }
    }
  }
  __syncthreads();   // every stage consumed: the ring becomes the reduction area
  // row-group blocks -> shared [warp][i][j][lane], then summed in warp order (element e = (i*NB+j)*32 + lane)
  float* red = ring;
  {
#pragma unroll
    for (int i = 0; i < MI; i++)
#pragma unroll
      for (int j = 0; j < NB; j++) red[((warp * MI + i) * NB + j) * 32 + lane] = (j & 1) ? acc[i][j / 2].y : acc[i][j / 2].x;
  }
  __syncthreads();
  auto coord = [&](int e, int& m, int& n) {   // tile element e -> output (m, n)
    const int ln = e & 31, ij = e >> 5, i = ij / NB, j = ij % NB;
    const int l = l0 + 32 * i + ln, q = q0 + j;
    if (p.trans) { m = q; n = l; } else { m = l; n = q; }
    return l < p.DL && q < p.DQ;
  };
  if (p.split == 1) {
    for (int e = tid; e < V; e += NTHR) {
      float v = 0.f;
#pragma unroll
      for (int w = 0; w < NCW; w++) v += red[w * V + e];
      int m, n;
      if (coord(e, m, n)) p.C[(long long)m * p.ldc + n] = v;
    }
  } else {
    const int ntile = p.tiles_l * p.tiles_q;
    float* part = p.part + (long long)tile * p.split * V;
    for (int e = tid; e < V; e += NTHR) {
      float v = 0.f;
#pragma unroll
      for (int w = 0; w < NCW; w++) v += red[w * V + e];
      part[(long long)z * V + e] = v;
    }
    __syncthreads();   // red is re-used below as the fp64 combine area
    double* out = reinterpret_cast<double*>(ring);
    double* scratch = out + V;
    const int ng = combine_rows(p.split);
    (void)ntile;
    if (combine_splits(p.tickets + tile * (1 + ng), part, p.gpart + (long long)tile * ng * V, V, p.split, z, V, out, scratch)) {
      for (int e = tid; e < V; e += NTHR) {
        int m, n;
        if (coord(e, m, n)) p.C[(long long)m * p.ldc + n] = (float)out[e];
      }
    }
  }
  orion_signal(sig);
}

typedef void (*kfn)(CUtensorMap, CUtensorMap, Params, OrionSig);

template <int MI, int NB>
const void* fn_ptr() { return (const void*)wgs_kernel<MI, NB>; }

inline const void* kernel_of(int mi, int nb) {
#define WGS_CASE(a, b) if (mi == a && nb == b) return fn_ptr<a, b>();
  WGS_CASE(1, 4) WGS_CASE(1, 8) WGS_CASE(1, 16) WGS_CASE(1, 24) WGS_CASE(1, 32)
  WGS_CASE(2, 4) WGS_CASE(2, 8) WGS_CASE(2, 16) WGS_CASE(2, 24) WGS_CASE(2, 32)
  WGS_CASE(3, 4) WGS_CASE(3, 8) WGS_CASE(3, 16) WGS_CASE(3, 24)
#undef WGS_CASE
  return nullptr;
}

inline bool prepare(const void* f, int smem) {
  // the largest smem any plan asks for is set once per kernel (all plans stay below it)
  (void)smem;
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  static const int MIS[3] = {1, 2, 3};
  static const int NBS[5] = {4, 8, 16, 24, 32};
  for (int mi : MIS)
    for (int nb : NBS) {
      const void* k = kernel_of(mi, nb);
      if (!k) continue;
      if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, STAGE_BUDGET + 4096) != cudaSuccess) {
        (void)cudaGetLastError();
        return false;
      }
    }
  (void)f;
  done.store(1, std::memory_order_release);
  return true;
}

}  // namespace wgs
}  // namespace

// ---- entry points used by gemm.cu (flags = 1 routing)
uint64_t wgs_ws_bytes(long long M, long long N, long long K) {
  if (M <= 0 || N <= 0 || K <= 0) return 0;
  return wgs::ws_bytes(wgs::plan(M, N, K));
}

// args: A, B, C, bias, M, N, K, lda, ldb, ldc, flags, workspace, ws_bytes
bool wgs_try_geom(const uint64_t* a, LaunchGeom* g) {
  const long long M = a[4], N = a[5], K = a[6], lda = a[7], ldb = a[8];
  const float* A = (const float*)a[0];
  const float* B = (const float*)a[1];
  if ((int)a[10] != 1 || a[3] != 0) return false;                 // A^T B without bias only
  if (K < 256 || lda % 4 || ldb % 4 || M % 4 || N % 4) return false;   // TMA strides / 16-byte boxes
  if (!tmah::al16(A) || !tmah::al16(B) || tmah::encoder() == nullptr) return false;
  if (M > (1 << 20) || N > (1 << 20) || K >= (1LL << 31)) return false;
  wgs::Plan pl = wgs::plan(M, N, K);
  if (pl.split > 1 && (a[11] == 0 || a[12] < wgs::ws_bytes(pl))) return false;
  if ((uint64_t)pl.tiles_l * pl.tiles_q * (1 + combine_rows(pl.split)) * 4 > WS_TICKET_BYTES) return false;
  const void* f = wgs::kernel_of(pl.mi, pl.nb);
  if (!f || !wgs::prepare(f, pl.smem)) return false;
  g->grid = dim3((unsigned)(pl.tiles_l * pl.tiles_q), (unsigned)pl.split);
  g->block = dim3(wgs::NTHR);
  g->smem = pl.smem;
  g->func = f;
  return true;
}

bool wgs_is(const void* f) {
  static const int MIS[3] = {1, 2, 3};
  static const int NBS[5] = {4, 8, 16, 24, 32};
  for (int mi : MIS)
    for (int nb : NBS)
      if (wgs::kernel_of(mi, nb) == f && f != nullptr) return true;
  return false;
}

int wgs_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  const long long M = a[4], N = a[5], K = a[6], lda = a[7], ldb = a[8], ldc = a[9];
  const float* A = (const float*)a[0];
  const float* B = (const float*)a[1];
  wgs::Plan pl = wgs::plan(M, N, K);
  wgs::Params p;
  p.trans = pl.trans;
  p.DL = (int)(pl.trans ? N : M); p.DQ = (int)(pl.trans ? M : N); p.K = (int)K;
  p.C = (float*)a[2]; p.ldc = ldc;
  p.tiles_l = pl.tiles_l; p.tiles_q = pl.tiles_q; p.split = pl.split; p.kps = pl.kps; p.R = pl.R; p.stages = pl.stages;
  p.tickets = nullptr; p.part = nullptr; p.gpart = nullptr;
  if (pl.split > 1) {
    unsigned char* ws = (unsigned char*)a[11];
    const uint64_t tiles = (uint64_t)pl.tiles_l * pl.tiles_q, V = 32ull * pl.mi * pl.nb;
    p.tickets = reinterpret_cast<unsigned int*>(ws);
    p.part = reinterpret_cast<float*>(ws + WS_TICKET_BYTES);
    uintptr_t gp = reinterpret_cast<uintptr_t>(ws + WS_TICKET_BYTES + tiles * pl.split * V * 4);
    gp = (gp + 15) & ~uintptr_t(15);
    p.gpart = reinterpret_cast<double*>(gp);
  }
  const float* Lb = pl.trans ? B : A;
  const float* Qb = pl.trans ? A : B;
  const long long ldL = pl.trans ? ldb : lda, ldQ = pl.trans ? lda : ldb;
  CUtensorMap mL, mQ;
  if (!tmah::map2d_f32(&mL, Lb, K, p.DL, ldL, 32 * pl.mi, pl.R)) return ORION_E_CUDA;
  if (!tmah::map2d_f32(&mQ, Qb, K, p.DQ, ldQ, pl.nb, pl.R)) return ORION_E_CUDA;
#define WGS_LAUNCH(a_, b_)                                                                          \
  if (pl.mi == a_ && pl.nb == b_) {                                                                 \
    wgs::wgs_kernel<a_, b_><<<g.grid, g.block, g.smem, s>>>(mL, mQ, p, sig);                        \
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;                                    \
  }
  WGS_LAUNCH(1, 4) WGS_LAUNCH(1, 8) WGS_LAUNCH(1, 16) WGS_LAUNCH(1, 24) WGS_LAUNCH(1, 32)
  WGS_LAUNCH(2, 4) WGS_LAUNCH(2, 8) WGS_LAUNCH(2, 16) WGS_LAUNCH(2, 24) WGS_LAUNCH(2, 32)
  WGS_LAUNCH(3, 4) WGS_LAUNCH(3, 8) WGS_LAUNCH(3, 16) WGS_LAUNCH(3, 24)
#undef WGS_LAUNCH
  return ORION_E_INVAL;
}
