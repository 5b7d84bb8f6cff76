// Dense GEMM and implicit-GEMM convolutions (fp32, FFMA tiles) with deterministic split-K.
//
// One tiled main loop serves Linear fwd/bwd (P:897-899 cuBLAS GEMM in the paper) and Conv2d
// fwd / dgrad / wgrad (cuDNN convolution) through operand "loaders" that map a GEMM
// coordinate to an address (im2col on the fly, NHWC activations, OHWI weights).
// Determinism: each output element is accumulated by one thread in k order; split-K partials are
// reduced by the last CTA of each tile in split order; the split count is a function of the
// shape only (never of the SM partition), so results are identical solo and collocated.
#include "common.cuh"

namespace {

constexpr int NT = 256;

// Tile configurations (shape-selected, never SM-count-selected). Thread grid is always 16 x 16;
// each thread owns a TM x TN sub-tile split in two halves (rows ty*TM/2.. and BM/2 + ty*TM/2..)
// to keep shared-memory fragment reads conflict-free. Every thread loads 4 A and 4 B elements
// per k-tile.
template <int BM_, int BN_, int BK_>
struct Tile {
  static constexpr int BM = BM_, BN = BN_, BK = BK_, TM = BM_ / 16, TN = BN_ / 16;
  static_assert(BM * BK == 4 * NT && BN * BK == 4 * NT, "4 loads per thread per operand");
};
using TileL = Tile<128, 128, 8>;   // 8x8 per thread: compute-dense problems
using TileM = Tile<64, 64, 16>;    // 4x4 per thread
using TileS = Tile<32, 32, 32>;    // 2x2 per thread: skinny / memory-bound (long-K wgrad)

struct GemmParams {
  int M, N, K;
  float* C;
  long long ldc;
  const float* bias;
  int split;           // number of K splits (grid.z)
  int kps;             // K elements per split (multiple of BK)
  float* ws;           // split partials [split][M][N] (split > 1)
  unsigned int* tickets;  // one per output tile (split > 1), zero at rest
};

// ---------------------------------------------------------------- operand loaders
// A(m, k) and B(k, n). kContigK says whether consecutive k are adjacent in memory; it picks the
// global->smem load mapping that keeps warps coalesced.
struct ADense {          // A row-major [M][lda]
  static constexpr bool kContigK = true;
  const float* p; long long ld;
  struct Row { long long base; bool ok; };
  __device__ Row row(int m, int M) const { return {(long long)m * ld, m < M}; }
  __device__ float at(const Row& r, int k, int K) const { return (r.ok && k < K) ? __ldg(p + r.base + k) : 0.f; }
};
struct ADenseT {         // A stored transposed: A(m,k) = p[k*ld + m]
  static constexpr bool kContigK = false;
  const float* p; long long ld;
  struct Row { int m; bool ok; };
  __device__ Row row(int m, int M) const { return {m, m < M}; }
  __device__ float at(const Row& r, int k, int K) const { return (r.ok && k < K) ? __ldg(p + (long long)k * ld + r.m) : 0.f; }
};
struct BDense {          // B row-major [K][ldb]: B(k,n) = p[k*ld + n]
  static constexpr bool kContigK = false;
  const float* p; long long ld;
  struct Col { int n; bool ok; };
  __device__ Col col(int n, int N) const { return {n, n < N}; }
  __device__ float at(const Col& c, int k, int K) const { return (c.ok && k < K) ? __ldg(p + (long long)k * ld + c.n) : 0.f; }
};
struct BDenseT {         // B stored transposed [N][ldb]: B(k,n) = p[n*ld + k]
  static constexpr bool kContigK = true;
  const float* p; long long ld;
  struct Col { long long base; bool ok; };
  __device__ Col col(int n, int N) const { return {(long long)n * ld, n < N}; }
  __device__ float at(const Col& c, int k, int K) const { return (c.ok && k < K) ? __ldg(p + c.base + k) : 0.f; }
};

struct ConvShape { int N, H, W, C, K, R, S, stride, pad, P, Q; };

// Conv fwd A: im2col of x. m = (n, p, q), k = (r, s, c) with c fastest (matches OHWI weights).
struct AIm2col {
  static constexpr bool kContigK = true;
  const float* x; ConvShape s;
  struct Row { long long nbase; int h0, w0; bool ok; };
  __device__ Row row(int m, int M) const {
    Row r; r.ok = m < M;
    int mm = r.ok ? m : 0;
    int q = mm % s.Q; int t = mm / s.Q; int p = t % s.P; int n = t / s.P;
    r.nbase = (long long)n * s.H * s.W * s.C; r.h0 = p * s.stride - s.pad; r.w0 = q * s.stride - s.pad;
    return r;
  }
  __device__ float at(const Row& r, int k, int K) const {
    if (!r.ok || k >= K) return 0.f;
    int c = k % s.C; int t = k / s.C; int ss = t % s.S; int rr = t / s.S;
    int h = r.h0 + rr, w = r.w0 + ss;
    if ((unsigned)h >= (unsigned)s.H || (unsigned)w >= (unsigned)s.W) return 0.f;
    return __ldg(x + r.nbase + ((long long)h * s.W + w) * s.C + c);
  }
};

// Conv dgrad A: m = (n, h, w) of dx, k = (r, s, kout) with kout fastest; A = dy[n, p, q, kout]
// where h = p*stride - pad + r.
struct ADgrad {
  static constexpr bool kContigK = true;
  const float* dy; ConvShape s;
  struct Row { long long nbase; int hp, wp; bool ok; };
  __device__ Row row(int m, int M) const {
    Row r; r.ok = m < M;
    int mm = r.ok ? m : 0;
    int w = mm % s.W; int t = mm / s.W; int h = t % s.H; int n = t / s.H;
    r.nbase = (long long)n * s.P * s.Q * s.K; r.hp = h + s.pad; r.wp = w + s.pad;
    return r;
  }
  __device__ float at(const Row& r, int k, int K) const {
    if (!r.ok || k >= K) return 0.f;
    int ko = k % s.K; int t = k / s.K; int ss = t % s.S; int rr = t / s.S;
    int ph = r.hp - rr, pw = r.wp - ss;
    if (ph < 0 || pw < 0 || ph % s.stride || pw % s.stride) return 0.f;
    int p = ph / s.stride, q = pw / s.stride;
    if (p >= s.P || q >= s.Q) return 0.f;
    return __ldg(dy + r.nbase + ((long long)p * s.Q + q) * s.K + ko);
  }
};
// Conv dgrad B: B(k = (r,s,kout), n = c) = w[kout][r][s][c]
struct BDgrad {
  static constexpr bool kContigK = false;
  const float* w; ConvShape s;
  struct Col { int c; bool ok; };
  __device__ Col col(int n, int N) const { return {n, n < N}; }
  __device__ float at(const Col& cc, int k, int K) const {
    if (!cc.ok || k >= K) return 0.f;
    int ko = k % s.K; int t = k / s.K; int ss = t % s.S; int rr = t / s.S;
    return __ldg(w + (((long long)ko * s.R + rr) * s.S + ss) * s.C + cc.c);
  }
};
// Conv wgrad B: B(k = (n,p,q), col = (r,s,c)) = x[n, p*st-pad+r, q*st-pad+s, c]
struct BWgrad {
  static constexpr bool kContigK = false;
  const float* x; ConvShape s;
  struct Col { int r, ss, c; bool ok; };
  __device__ Col col(int n, int N) const {
    Col cc; cc.ok = n < N; int nn = cc.ok ? n : 0;
    cc.c = nn % s.C; int t = nn / s.C; cc.ss = t % s.S; cc.r = t / s.S;
    return cc;
  }
  __device__ float at(const Col& cc, int k, int K) const {
    if (!cc.ok || k >= K) return 0.f;
    int q = k % s.Q; int t = k / s.Q; int p = t % s.P; int n = t / s.P;
    int h = p * s.stride - s.pad + cc.r, w = q * s.stride - s.pad + cc.ss;
    if ((unsigned)h >= (unsigned)s.H || (unsigned)w >= (unsigned)s.W) return 0.f;
    return __ldg(x + (((long long)n * s.H + h) * s.W + w) * s.C + cc.c);
  }
};

// ---------------------------------------------------------------- the tiled main loop
template <int N_>
__device__ __forceinline__ void lds_frag(float* dst, const float* src) {
  if constexpr (N_ == 4) {
    float4 v = *reinterpret_cast<const float4*>(src);
    dst[0] = v.x; dst[1] = v.y; dst[2] = v.z; dst[3] = v.w;
  } else if constexpr (N_ == 2) {
    float2 v = *reinterpret_cast<const float2*>(src);
    dst[0] = v.x; dst[1] = v.y;
  } else {
    dst[0] = *src;
  }
}

template <class T, class LA, class LB>
__global__ void __launch_bounds__(NT) gemm_kernel(GemmParams p, LA la, LB lb, OrionSig sig) {
  constexpr int BM = T::BM, BN = T::BN, BK = T::BK, TM = T::TM, TN = T::TN;
  __shared__ __align__(16) float As[2][BK][BM + 4];
  __shared__ __align__(16) float Bs[2][BK][BN + 4];
  const int tid = threadIdx.x;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  const int kbeg = blockIdx.z * p.kps;
  const int kend = min(p.K, kbeg + p.kps);

  int a_m[4], a_k[4], b_n[4], b_k[4];
#pragma unroll
  for (int i = 0; i < 4; i++) {
    if (LA::kContigK) { a_k[i] = tid % BK; a_m[i] = tid / BK + (NT / BK) * i; }
    else { a_m[i] = tid % BM; a_k[i] = tid / BM + (NT / BM) * i; }
    if (LB::kContigK) { b_k[i] = tid % BK; b_n[i] = tid / BK + (NT / BK) * i; }
    else { b_n[i] = tid % BN; b_k[i] = tid / BN + (NT / BN) * i; }
  }
  typename LA::Row arow[4];
  typename LB::Col bcol[4];
#pragma unroll
  for (int i = 0; i < 4; i++) { arow[i] = la.row(m0 + a_m[i], p.M); bcol[i] = lb.col(n0 + b_n[i], p.N); }

  float ra[4], rb[4];
  auto gload = [&](int k0) {
#pragma unroll
    for (int i = 0; i < 4; i++) {
      int ka = k0 + a_k[i], kb = k0 + b_k[i];
      ra[i] = ka < kend ? la.at(arow[i], ka, p.K) : 0.f;
      rb[i] = kb < kend ? lb.at(bcol[i], kb, p.K) : 0.f;
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int i = 0; i < 4; i++) { As[buf][a_k[i]][a_m[i]] = ra[i]; Bs[buf][b_k[i]][b_n[i]] = rb[i]; }
  };

  float acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; i++)
#pragma unroll
    for (int j = 0; j < TN; j++) acc[i][j] = 0.f;

  const int ty = tid / 16, tx = tid % 16;
  int buf = 0;
  if (kbeg < kend) {
    gload(kbeg);
    sstore(0);
  }
  __syncthreads();
  for (int k0 = kbeg; k0 < kend; k0 += BK) {
    const bool more = k0 + BK < kend;
    if (more) gload(k0 + BK);
#pragma unroll
    for (int kk = 0; kk < BK; kk++) {
      float av[TM], bv[TN];
      lds_frag<TM / 2>(av, &As[buf][kk][ty * (TM / 2)]);
      lds_frag<TM / 2>(av + TM / 2, &As[buf][kk][BM / 2 + ty * (TM / 2)]);
      lds_frag<TN / 2>(bv, &Bs[buf][kk][tx * (TN / 2)]);
      lds_frag<TN / 2>(bv + TN / 2, &Bs[buf][kk][BN / 2 + tx * (TN / 2)]);
#pragma unroll
      for (int i = 0; i < TM; i++)
#pragma unroll
        for (int j = 0; j < TN; j++) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    if (more) {
      sstore(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }

  auto out_row = [&](int i) { return m0 + (i < TM / 2 ? ty * (TM / 2) + i : BM / 2 + ty * (TM / 2) + (i - TM / 2)); };
  auto out_col = [&](int j) { return n0 + (j < TN / 2 ? tx * (TN / 2) + j : BN / 2 + tx * (TN / 2) + (j - TN / 2)); };
  if (p.split == 1) {
#pragma unroll
    for (int i = 0; i < TM; i++) {
      int m = out_row(i);
      if (m >= p.M) continue;
#pragma unroll
      for (int j = 0; j < TN; j++) {
        int n = out_col(j);
        if (n < p.N) p.C[(long long)m * p.ldc + n] = acc[i][j] + (p.bias ? __ldg(p.bias + n) : 0.f);
      }
    }
  } else {
    float* part = p.ws + (long long)blockIdx.z * p.M * p.N;
#pragma unroll
    for (int i = 0; i < TM; i++) {
      int m = out_row(i);
      if (m >= p.M) continue;
#pragma unroll
      for (int j = 0; j < TN; j++) {
        int n = out_col(j);
        if (n < p.N) part[(long long)m * p.N + n] = acc[i][j];
      }
    }
    unsigned int* tk = p.tickets + blockIdx.y * gridDim.x + blockIdx.x;
    if (last_cta_of(tk, p.split)) {
#pragma unroll
      for (int i = 0; i < TM; i++) {
        int m = out_row(i);
        if (m >= p.M) continue;
#pragma unroll
        for (int j = 0; j < TN; j++) {
          int n = out_col(j);
          if (n >= p.N) continue;
          float s = 0.f;
          for (int z = 0; z < p.split; z++) s += __ldcg(p.ws + (long long)z * p.M * p.N + (long long)m * p.N + n);
          p.C[(long long)m * p.ldc + n] = s + (p.bias ? __ldg(p.bias + n) : 0.f);
        }
      }
    }
  }
  orion_signal(sig);
}

// ---------------------------------------------------------------- small-M GEMM (GEMV-like)
// For M <= 8 with B transposed (weights [N][K], the Linear layout): one warp per output column n,
// lanes stride k with float4 loads; all M rows at once; fixed shuffle-tree reduction.
constexpr int SM_MAXM = 8;
__global__ void __launch_bounds__(256) gemv_bt_kernel(const float* __restrict__ A, long long lda,
                                                      const float* __restrict__ B, long long ldb,
                                                      float* __restrict__ C, long long ldc,
                                                      const float* __restrict__ bias, int M, int N, int K,
                                                      OrionSig sig) {
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int n = blockIdx.x * 8 + warp;
  float acc[SM_MAXM];
#pragma unroll
  for (int i = 0; i < SM_MAXM; i++) acc[i] = 0.f;
  if (n < N) {
    const float* brow = B + (long long)n * ldb;
    const bool vec = ((K & 3) == 0) && ((lda & 3) == 0) && ((ldb & 3) == 0) &&
                     ((reinterpret_cast<uintptr_t>(A) & 15) == 0) && ((reinterpret_cast<uintptr_t>(B) & 15) == 0);
    if (vec) {
      for (int k = lane * 4; k < K; k += 128) {
        float4 b = __ldg(reinterpret_cast<const float4*>(brow + k));
#pragma unroll
        for (int i = 0; i < SM_MAXM; i++) {
          if (i < M) {
            float4 a = __ldg(reinterpret_cast<const float4*>(A + (long long)i * lda + k));
            acc[i] = fmaf(a.x, b.x, acc[i]); acc[i] = fmaf(a.y, b.y, acc[i]);
            acc[i] = fmaf(a.z, b.z, acc[i]); acc[i] = fmaf(a.w, b.w, acc[i]);
          }
        }
      }
    } else {
      for (int k = lane; k < K; k += 32) {
        float b = __ldg(brow + k);
#pragma unroll
        for (int i = 0; i < SM_MAXM; i++)
          if (i < M) acc[i] = fmaf(__ldg(A + (long long)i * lda + k), b, acc[i]);
      }
    }
#pragma unroll
    for (int i = 0; i < SM_MAXM; i++)
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], o);
    if (lane == 0) {
      float b = bias ? __ldg(bias + n) : 0.f;
#pragma unroll
      for (int i = 0; i < SM_MAXM; i++)
        if (i < M) C[(long long)i * ldc + n] = acc[i] + b;
    }
  }
  orion_signal(sig);
}

// Shape-only plan: tile config and K split. Splits target ~4 waves of 148 SMs (a constant of the
// part's size class, never the partition's SM count) so long-K problems (weight gradients over
// N*H*W rows, 3x3 convs at batch 4) spread over the GPU; the split reduction is ordered.
struct Plan { int cfg; int split; int bm, bn, bk; };

Plan plan_gemm(long long M, long long N, long long K) {
  Plan pl;
  if (M >= 128 && N >= 128 && M * N >= 128LL * 128 * 64) { pl.cfg = 0; pl.bm = 128; pl.bn = 128; pl.bk = 8; }
  else if (M >= 48 && N >= 48) { pl.cfg = 1; pl.bm = 64; pl.bn = 64; pl.bk = 16; }
  else { pl.cfg = 2; pl.bm = 32; pl.bn = 32; pl.bk = 32; }
  long long tiles = cdiv(M, pl.bm) * cdiv(N, pl.bn);
  long long target = 592;
  long long split = 1;
  if (tiles < target) {
    split = cdiv(target, tiles);
    long long kmax = K / (4 * pl.bk);         // >= 4 k-tiles per split
    if (split > kmax) split = kmax;
    if (split > 512) split = 512;
    if (split < 1) split = 1;
  }
  pl.split = (int)split;
  return pl;
}

uint64_t ws_bytes_for(const Plan& pl, long long M, long long N) {
  return pl.split > 1 ? WS_TICKET_BYTES + (uint64_t)pl.split * M * N * 4 : 0;
}

template <class LA, class LB>
const void* kernel_for(int cfg) {
  switch (cfg) {
    case 0: return (const void*)gemm_kernel<TileL, LA, LB>;
    case 1: return (const void*)gemm_kernel<TileM, LA, LB>;
    default: return (const void*)gemm_kernel<TileS, LA, LB>;
  }
}

// Geometry of a tiled launch; falls back to split 1 when the caller's workspace is too small.
template <class LA, class LB>
void tiled_geom(LaunchGeom* g, long long M, long long N, long long K, uint64_t ws_ptr, uint64_t ws_bytes) {
  Plan pl = plan_gemm(M, N, K);
  if (pl.split > 1 && (ws_ptr == 0 || ws_bytes < ws_bytes_for(pl, M, N))) pl.split = 1;
  g->grid = dim3((unsigned)cdiv(N, pl.bn), (unsigned)cdiv(M, pl.bm), (unsigned)pl.split);
  g->block = dim3(NT);
  g->smem = 0;
  g->func = kernel_for<LA, LB>(pl.cfg);
}

GemmParams make_params(long long M, long long N, long long K, float* C, long long ldc, const float* bias, int split,
                       float* ws, int bk) {
  GemmParams p;
  p.M = (int)M; p.N = (int)N; p.K = (int)K; p.C = C; p.ldc = ldc; p.bias = bias;
  p.split = split;
  p.kps = (int)(cdiv(cdiv(K, split), bk) * bk);
  p.ws = nullptr;
  p.tickets = nullptr;
  if (split > 1) {  // workspace layout: [tickets (WS_TICKET_BYTES)][partials]
    p.tickets = reinterpret_cast<unsigned int*>(ws);
    p.ws = reinterpret_cast<float*>(reinterpret_cast<char*>(ws) + WS_TICKET_BYTES);
  }
  return p;
}

template <class LA, class LB>
int launch_tiled(const LaunchGeom& g, long long M, long long N, long long K, float* C, long long ldc, const float* bias,
                 float* ws, LA la, LB lb, OrionSig sig, cudaStream_t s) {
  const int split = (int)g.grid.z;
  if (g.func == (const void*)gemm_kernel<TileL, LA, LB>) {
    gemm_kernel<TileL, LA, LB><<<g.grid, g.block, 0, s>>>(make_params(M, N, K, C, ldc, bias, split, ws, TileL::BK), la, lb, sig);
  } else if (g.func == (const void*)gemm_kernel<TileM, LA, LB>) {
    gemm_kernel<TileM, LA, LB><<<g.grid, g.block, 0, s>>>(make_params(M, N, K, C, ldc, bias, split, ws, TileM::BK), la, lb, sig);
  } else {
    gemm_kernel<TileS, LA, LB><<<g.grid, g.block, 0, s>>>(make_params(M, N, K, C, ldc, bias, split, ws, TileS::BK), la, lb, sig);
  }
  return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
}

}  // namespace

// Workspace bytes a tiled GEMM of this (M, N, K) needs for its K split (0 if no split). Conv ops
// pass their implicit-GEMM dims: fwd (N*P*Q, K, R*S*C), dgrad (N*H*W, C, R*S*K), wgrad (K, R*S*C, N*P*Q).
extern "C" uint64_t orion_gemm_workspace_bytes(uint64_t M, uint64_t N, uint64_t K) {
  Plan pl = plan_gemm((long long)M, (long long)N, (long long)K);
  return ws_bytes_for(pl, (long long)M, (long long)N);
}

// ------------------------------------------------------------------------- GEMM entry
// args: A, B, C, bias, M, N, K, lda, ldb, ldc, flags(1=A^T, 2=B^T), workspace, ws_bytes
int gemm_geom(const uint64_t* a, LaunchGeom* g) {
  long long M = a[4], N = a[5], K = a[6];
  int flags = (int)a[10];
  if (M <= 0 || N <= 0 || K <= 0) return ORION_E_INVAL;
  if (M <= SM_MAXM && flags == 2) {
    g->grid = dim3((unsigned)cdiv(N, 8)); g->block = dim3(256); g->smem = 0; g->func = (const void*)gemv_bt_kernel;
    return 0;
  }
  switch (flags) {
    case 0: tiled_geom<ADense, BDense>(g, M, N, K, a[11], a[12]); break;
    case 1: tiled_geom<ADenseT, BDense>(g, M, N, K, a[11], a[12]); break;
    case 2: tiled_geom<ADense, BDenseT>(g, M, N, K, a[11], a[12]); break;
    case 3: tiled_geom<ADenseT, BDenseT>(g, M, N, K, a[11], a[12]); break;
    default: return ORION_E_INVAL;
  }
  return 0;
}

int gemm_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  const float* A = (const float*)a[0];
  const float* B = (const float*)a[1];
  float* C = (float*)a[2];
  const float* bias = (const float*)a[3];
  long long M = a[4], N = a[5], K = a[6], lda = a[7], ldb = a[8], ldc = a[9];
  int flags = (int)a[10];
  float* ws = (float*)a[11];
  if (g.func == (const void*)gemv_bt_kernel) {
    gemv_bt_kernel<<<g.grid, g.block, 0, s>>>(A, lda, B, ldb, C, ldc, bias, (int)M, (int)N, (int)K, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  switch (flags) {
    case 0: return launch_tiled(g, M, N, K, C, ldc, bias, ws, ADense{A, lda}, BDense{B, ldb}, sig, s);
    case 1: return launch_tiled(g, M, N, K, C, ldc, bias, ws, ADenseT{A, lda}, BDense{B, ldb}, sig, s);
    case 2: return launch_tiled(g, M, N, K, C, ldc, bias, ws, ADense{A, lda}, BDenseT{B, ldb}, sig, s);
    case 3: return launch_tiled(g, M, N, K, C, ldc, bias, ws, ADenseT{A, lda}, BDenseT{B, ldb}, sig, s);
  }
  return ORION_E_INVAL;
}

// ------------------------------------------------------------------------- convolutions
// args: x|dy, w|dy, y|dx|dw, N, H, W, C, K, R, S, stride, pad, P, Q, workspace, ws_bytes
static ConvShape conv_shape(const uint64_t* a) {
  ConvShape s;
  s.N = (int)a[3]; s.H = (int)a[4]; s.W = (int)a[5]; s.C = (int)a[6]; s.K = (int)a[7];
  s.R = (int)a[8]; s.S = (int)a[9]; s.stride = (int)a[10]; s.pad = (int)a[11]; s.P = (int)a[12]; s.Q = (int)a[13];
  return s;
}

// implicit-GEMM dims: fwd (M = N*P*Q, N = K, K = R*S*C); dgrad (N*H*W, C, R*S*K); wgrad (K, R*S*C, N*P*Q)
int conv_fwd_geom(const uint64_t* a, LaunchGeom* g) {
  ConvShape s = conv_shape(a);
  tiled_geom<AIm2col, BDenseT>(g, (long long)s.N * s.P * s.Q, s.K, (long long)s.R * s.S * s.C, a[14], a[15]);
  return 0;
}
int conv_fwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  ConvShape s = conv_shape(a);
  long long M = (long long)s.N * s.P * s.Q, N = s.K, K = (long long)s.R * s.S * s.C;
  return launch_tiled(g, M, N, K, (float*)a[2], N, nullptr, (float*)a[14], AIm2col{(const float*)a[0], s},
                      BDenseT{(const float*)a[1], K}, sig, st);
}

int conv_dgrad_geom(const uint64_t* a, LaunchGeom* g) {
  ConvShape s = conv_shape(a);
  tiled_geom<ADgrad, BDgrad>(g, (long long)s.N * s.H * s.W, s.C, (long long)s.R * s.S * s.K, a[14], a[15]);
  return 0;
}
int conv_dgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  ConvShape s = conv_shape(a);
  long long M = (long long)s.N * s.H * s.W, N = s.C, K = (long long)s.R * s.S * s.K;
  return launch_tiled(g, M, N, K, (float*)a[2], N, nullptr, (float*)a[14], ADgrad{(const float*)a[0], s},
                      BDgrad{(const float*)a[1], s}, sig, st);
}

int conv_wgrad_geom(const uint64_t* a, LaunchGeom* g) {
  ConvShape s = conv_shape(a);
  tiled_geom<ADenseT, BWgrad>(g, s.K, (long long)s.R * s.S * s.C, (long long)s.N * s.P * s.Q, a[14], a[15]);
  return 0;
}
int conv_wgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  ConvShape s = conv_shape(a);
  long long M = s.K, N = (long long)s.R * s.S * s.C, K = (long long)s.N * s.P * s.Q;
  // A(m = kout, k = npq) = dy[npq * K + kout]
  return launch_tiled(g, M, N, K, (float*)a[2], N, nullptr, (float*)a[14], ADenseT{(const float*)a[1], s.K},
                      BWgrad{(const float*)a[0], s}, sig, st);
}
