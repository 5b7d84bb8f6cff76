// Dense GEMM and implicit-GEMM convolutions (fp32, FFMA tiles) with deterministic split-K.
//
// One tiled main loop serves Linear fwd/bwd (P:897-899 cuBLAS GEMM in the paper) and Conv2d
// fwd / dgrad / wgrad (cuDNN convolution) through operand "loaders" that map a GEMM
// coordinate to an address (im2col on the fly, NHWC activations, OHWI weights).
// Determinism: each output element is accumulated by one thread in k order; split-K partials are
// reduced by the last CTA of each tile in split order; the split count is a function of the
// shape only (never of the SM partition), so results are identical solo and collocated.
#include <atomic>
#include <cstdlib>

#include <cuda.h>

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
// at4(r, k, kend): the 4 values at k..k+3 (k % 4 == 0), zero beyond kend; one 128-bit load when the
// 4 are contiguous and aligned, else 4 scalar loads.
__device__ __forceinline__ bool al16(const float* q) { return (reinterpret_cast<uintptr_t>(q) & 15) == 0; }

// Per-k-tile address helpers for the tensor-core producer: tile(k0, kend, bk) precomputes what is
// uniform over the tile (a conv tap when the tile lies inside one tap's channels); quad(row, t,
// kq, kend, q) then resolves quad kq of the tile for one row with a few adds. Loaders without a
// fast path fall back to addr4 / addr.
struct NoTile { int k0; };

struct ADense {          // A row-major [M][lda]
  static constexpr bool kContigK = true;
  const float* p; long long ld;
  struct Row { long long base; bool ok; };
  __device__ Row row(int m, int M) const { return {(long long)m * ld, m < M}; }
  __device__ float at(const Row& r, int k, int K) const { return (r.ok && k < K) ? __ldg(p + r.base + k) : 0.f; }
  // address of element k (nullptr = zero) and of an aligned contiguous quad (true + ptr/nullptr)
  __device__ const float* addr(const Row& r, int k, int kend) const { return (r.ok && k < kend) ? p + r.base + k : nullptr; }
  __device__ bool addr4(const Row& r, int k, int kend, const float*& q) const {
    if (!r.ok || k >= kend) { q = nullptr; return true; }
    q = p + r.base + k;
    return k + 3 < kend && al16(q);
  }
  __device__ NoTile tile(int k0, int, int) const { return {k0}; }
  template <class RC>
  __device__ bool quad(const RC& r, const NoTile& t, int kq, int kend, const float*& q) const { return addr4(r, t.k0 + 4 * kq, kend, q); }
};
struct ADenseT {         // A stored transposed: A(m,k) = p[k*ld + m]
  static constexpr bool kContigK = false;
  const float* p; long long ld;
  struct Row { int m; bool ok; };
  __device__ Row row(int m, int M) const { return {m, m < M}; }
  __device__ float at(const Row& r, int k, int K) const { return (r.ok && k < K) ? __ldg(p + (long long)k * ld + r.m) : 0.f; }
  __device__ const float* addr(const Row& r, int k, int kend) const { return (r.ok && k < kend) ? p + (long long)k * ld + r.m : nullptr; }
  __device__ bool addr4(const Row& r, int k, int kend, const float*& q) const {
    if (!r.ok || k >= kend) { q = nullptr; return true; }
    return false;
  }
  __device__ NoTile tile(int k0, int, int) const { return {k0}; }
  template <class RC>
  __device__ bool quad(const RC& r, const NoTile& t, int kq, int kend, const float*& q) const { return addr4(r, t.k0 + 4 * kq, kend, q); }
};
struct BDense {          // B row-major [K][ldb]: B(k,n) = p[k*ld + n]
  static constexpr bool kContigK = false;
  const float* p; long long ld;
  struct Col { int n; bool ok; };
  __device__ Col col(int n, int N) const { return {n, n < N}; }
  __device__ float at(const Col& c, int k, int K) const { return (c.ok && k < K) ? __ldg(p + (long long)k * ld + c.n) : 0.f; }
  __device__ const float* addr(const Col& c, int k, int kend) const { return (c.ok && k < kend) ? p + (long long)k * ld + c.n : nullptr; }
  __device__ bool addr4(const Col& c, int k, int kend, const float*& q) const {
    if (!c.ok || k >= kend) { q = nullptr; return true; }
    return false;
  }
  __device__ NoTile tile(int k0, int, int) const { return {k0}; }
  template <class RC>
  __device__ bool quad(const RC& r, const NoTile& t, int kq, int kend, const float*& q) const { return addr4(r, t.k0 + 4 * kq, kend, q); }
};
struct BDenseT {         // B stored transposed [N][ldb]: B(k,n) = p[n*ld + k]
  static constexpr bool kContigK = true;
  const float* p; long long ld;
  struct Col { long long base; bool ok; };
  __device__ Col col(int n, int N) const { return {(long long)n * ld, n < N}; }
  __device__ float at(const Col& c, int k, int K) const { return (c.ok && k < K) ? __ldg(p + c.base + k) : 0.f; }
  __device__ const float* addr(const Col& c, int k, int kend) const { return (c.ok && k < kend) ? p + c.base + k : nullptr; }
  __device__ bool addr4(const Col& c, int k, int kend, const float*& q) const {
    if (!c.ok || k >= kend) { q = nullptr; return true; }
    q = p + c.base + k;
    return k + 3 < kend && al16(q);
  }
  __device__ NoTile tile(int k0, int, int) const { return {k0}; }
  template <class RC>
  __device__ bool quad(const RC& r, const NoTile& t, int kq, int kend, const float*& q) const { return addr4(r, t.k0 + 4 * kq, kend, q); }
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
  __device__ const float* addr(const Row& r, int k, int kend) const {
    if (!r.ok || k >= kend) return nullptr;
    int c = k % s.C; int t = k / s.C; int ss = t % s.S; int rr = t / s.S;
    int h = r.h0 + rr, w = r.w0 + ss;
    if ((unsigned)h >= (unsigned)s.H || (unsigned)w >= (unsigned)s.W) return nullptr;
    return x + r.nbase + ((long long)h * s.W + w) * s.C + c;
  }
  __device__ bool addr4(const Row& r, int k, int kend, const float*& q) const {
    if (!r.ok || k >= kend) { q = nullptr; return true; }
    if ((s.C & 3) != 0 || k + 3 >= kend) return false;
    q = addr(r, k, kend);   // same tap for the 4 channels; nullptr = padding
    return q == nullptr || al16(q);
  }
  // tile inside one tap (C % bk == 0): every row's quad kq is 4 consecutive channels at one pixel
  struct Tile { int k0, rr, ss, c0; bool fast; };
  __device__ Tile tile(int k0, int kend, int bk) const {
    Tile t; t.k0 = k0; t.fast = (s.C % bk) == 0 && k0 + bk <= kend;
    int c = k0 % s.C, u = k0 / s.C; t.c0 = c; t.ss = u % s.S; t.rr = u / s.S;
    return t;
  }
  __device__ bool quad(const Row& r, const Tile& t, int kq, int kend, const float*& q) const {
    if (!t.fast) return addr4(r, t.k0 + 4 * kq, kend, q);
    const int h = r.h0 + t.rr, w = r.w0 + t.ss;
    if (!r.ok || (unsigned)h >= (unsigned)s.H || (unsigned)w >= (unsigned)s.W) { q = nullptr; return true; }
    q = x + r.nbase + ((long long)h * s.W + w) * s.C + t.c0 + 4 * kq;
    return al16(q);
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
  __device__ const float* addr(const Row& r, int k, int kend) const {
    if (!r.ok || k >= kend) return nullptr;
    int ko = k % s.K; int t = k / s.K; int ss = t % s.S; int rr = t / s.S;
    int ph = r.hp - rr, pw = r.wp - ss;
    if (ph < 0 || pw < 0 || ph % s.stride || pw % s.stride) return nullptr;
    int p = ph / s.stride, q = pw / s.stride;
    if (p >= s.P || q >= s.Q) return nullptr;
    return dy + r.nbase + ((long long)p * s.Q + q) * s.K + ko;
  }
  __device__ bool addr4(const Row& r, int k, int kend, const float*& q) const {
    if (!r.ok || k >= kend) { q = nullptr; return true; }
    if ((s.K & 3) != 0 || k + 3 >= kend) return false;
    q = addr(r, k, kend);
    return q == nullptr || al16(q);
  }
  struct Tile { int k0, rr, ss, ko0; bool fast; };
  __device__ Tile tile(int k0, int kend, int bk) const {
    Tile t; t.k0 = k0; t.fast = (s.K % bk) == 0 && k0 + bk <= kend;
    int c = k0 % s.K, u = k0 / s.K; t.ko0 = c; t.ss = u % s.S; t.rr = u / s.S;
    return t;
  }
  __device__ bool quad(const Row& r, const Tile& t, int kq, int kend, const float*& q) const {
    if (!t.fast) return addr4(r, t.k0 + 4 * kq, kend, q);
    const int ph = r.hp - t.rr, pw = r.wp - t.ss;
    if (!r.ok || ph < 0 || pw < 0 || ph % s.stride || pw % s.stride) { q = nullptr; return true; }
    const int p = ph / s.stride, qq = pw / s.stride;
    if (p >= s.P || qq >= s.Q) { q = nullptr; return true; }
    q = dy + r.nbase + ((long long)p * s.Q + qq) * s.K + t.ko0 + 4 * kq;
    return al16(q);
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
  __device__ const float* addr(const Col& cc, int k, int kend) const {
    if (!cc.ok || k >= kend) return nullptr;
    int ko = k % s.K; int t = k / s.K; int ss = t % s.S; int rr = t / s.S;
    return w + (((long long)ko * s.R + rr) * s.S + ss) * s.C + cc.c;
  }
  __device__ bool addr4(const Col& c, int k, int kend, const float*& q) const {
    if (!c.ok || k >= kend) { q = nullptr; return true; }
    return false;
  }
  __device__ NoTile tile(int k0, int, int) const { return {k0}; }
  template <class RC>
  __device__ bool quad(const RC& r, const NoTile& t, int kq, int kend, const float*& q) const { return addr4(r, t.k0 + 4 * kq, kend, q); }
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
  __device__ const float* addr(const Col& cc, int k, int kend) const {
    if (!cc.ok || k >= kend) return nullptr;
    int q = k % s.Q; int t = k / s.Q; int p = t % s.P; int n = t / s.P;
    int h = p * s.stride - s.pad + cc.r, w = q * s.stride - s.pad + cc.ss;
    if ((unsigned)h >= (unsigned)s.H || (unsigned)w >= (unsigned)s.W) return nullptr;
    return x + (((long long)n * s.H + h) * s.W + w) * s.C + cc.c;
  }
  __device__ bool addr4(const Col& c, int k, int kend, const float*& q) const {
    if (!c.ok || k >= kend) { q = nullptr; return true; }
    return false;
  }
  __device__ NoTile tile(int k0, int, int) const { return {k0}; }
  template <class RC>
  __device__ bool quad(const RC& r, const NoTile& t, int kq, int kend, const float*& q) const { return addr4(r, t.k0 + 4 * kq, kend, q); }
};

// ---------------------------------------------------------------- ordered split-K reduction
// dst[m0:m0+bm, n0:n0+bn] = sum_{z < count} src[z] (+ bias), summed in z order (((s0 + s1) + s2) + ...)
// by every thread of the calling CTA: consecutive threads on consecutive columns (coalesced),
// 128-bit where possible, 4 partials in flight.
__device__ void reduce_range(const float* src, long long zstride, int count, float* dst, long long ldd, const float* bias,
                             int M, int N, int m0, int n0, int bm, int bn) {
  const int rows = min(bm, M - m0), cols = min(bn, N - n0);
  const bool vec = (cols % 4 == 0) && (N % 4 == 0) && (n0 % 4 == 0) && (ldd % 4 == 0) &&
                   ((reinterpret_cast<uintptr_t>(src) & 15) == 0) && ((reinterpret_cast<uintptr_t>(dst) & 15) == 0) &&
                   (zstride % 4 == 0);
  if (vec) {
    const int cq = cols / 4, total = rows * cq;
    for (int e = threadIdx.x; e < total; e += blockDim.x) {
      const int r = e / cq, c = (e % cq) * 4;
      const float* q = src + (long long)(m0 + r) * N + n0 + c;
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
      int z = 0;
      for (; z + 7 < count; z += 8) {
        float4 v[8];
#pragma unroll
        for (int i = 0; i < 8; i++) v[i] = __ldcg(reinterpret_cast<const float4*>(q + (z + i) * zstride));
#pragma unroll
        for (int i = 0; i < 8; i++) { acc.x += v[i].x; acc.y += v[i].y; acc.z += v[i].z; acc.w += v[i].w; }
      }
      for (; z < count; z++) {
        float4 v = __ldcg(reinterpret_cast<const float4*>(q + z * zstride));
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
      }
      const int n = n0 + c;
      if (bias) {
        acc.x += __ldg(bias + n); acc.y += __ldg(bias + n + 1); acc.z += __ldg(bias + n + 2); acc.w += __ldg(bias + n + 3);
      }
      *reinterpret_cast<float4*>(dst + (long long)(m0 + r) * ldd + n) = acc;
    }
  } else {
    const int total = rows * cols;
    for (int e = threadIdx.x; e < total; e += blockDim.x) {
      const int r = e / cols, c = e % cols;
      const float* q = src + (long long)(m0 + r) * N + n0 + c;
      float acc = 0.f;
      int z = 0;
      for (; z + 3 < count; z += 4) {
        float v0 = __ldcg(q + z * zstride), v1 = __ldcg(q + (z + 1) * zstride);
        float v2 = __ldcg(q + (z + 2) * zstride), v3 = __ldcg(q + (z + 3) * zstride);
        acc += v0; acc += v1; acc += v2; acc += v3;
      }
      for (; z < count; z++) acc += __ldcg(q + z * zstride);
      dst[(long long)(m0 + r) * ldd + n0 + c] = acc + (bias ? __ldg(bias + n0 + c) : 0.f);
    }
  }
}

// Finish a split-K tile after this CTA wrote its partial p.ws[blockIdx.z]. Up to 32 splits: the
// last CTA of the tile sums all partials in order. More: a fixed two-level tree — the last CTA of
// each group of 16 consecutive splits sums the group into a group partial (after the split
// partials in the workspace), and the last group to finish sums the group partials in order.
// The group size is ~sqrt(split) (combine_group: both levels sum ~sqrt(split) partials).
constexpr int SPLIT_FLAT_MAX = 32, TICKETS_PER_TILE = 64;
__host__ __device__ __forceinline__ int split_groups(int split) {   // group partials (0: flat)
  return split <= SPLIT_FLAT_MAX ? 0 : (split + combine_group(split) - 1) / combine_group(split);
}
__device__ void split_finish(const GemmParams& p, int tile, int m0, int n0, int bm, int bn) {
  const long long MN = (long long)p.M * p.N;
  if (p.split <= SPLIT_FLAT_MAX) {
    if (last_cta_of(p.tickets + tile, p.split)) reduce_range(p.ws, MN, p.split, p.C, p.ldc, p.bias, p.M, p.N, m0, n0, bm, bn);
    return;
  }
  const int SPLIT_GROUP = combine_group(p.split);
  const int ng = (p.split + SPLIT_GROUP - 1) / SPLIT_GROUP;
  const int g = blockIdx.z / SPLIT_GROUP;
  const int gsize = min(SPLIT_GROUP, p.split - g * SPLIT_GROUP);
  unsigned int* tb = p.tickets + (long long)tile * TICKETS_PER_TILE;
  float* gws = p.ws + (long long)p.split * MN;
  if (last_cta_of(tb + 1 + g, gsize)) {
    reduce_range(p.ws + (long long)g * SPLIT_GROUP * MN, MN, gsize, gws + (long long)g * MN, p.N, nullptr, p.M, p.N, m0, n0, bm, bn);
    if (last_cta_of(tb, ng)) reduce_range(gws, MN, ng, p.C, p.ldc, p.bias, p.M, p.N, m0, n0, bm, bn);
  }
}

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
    split_finish(p, blockIdx.y * gridDim.x + blockIdx.x, m0, n0, BM, BN);
  }
  orion_signal(sig);
}

// ---------------------------------------------------------------- tcgen05 path (sm_100a)
// fp32 GEMM on the 5th-generation tensor cores with a 3xTF32 split: every operand
// x = hi + lo with hi = rna_tf32(x), lo = x - hi, and D += A_lo B_hi + A_hi B_lo + A_hi B_hi per
// k-step (kind::tf32, fp32 accumulators in TMEM). This keeps fp32-level accuracy (~2^-21 relative
// per product) where plain TF32 would miss the 1e-4 parity bar.
// Warp roles (160 threads): warps 0-3 stage operands (loader -> hi/lo split -> UMMA K-major
// SWIZZLE_NONE core-matrix layout in shared memory) and later run the epilogue (TMEM lanes
// 32w..32w+31 -> registers -> global); warp 4 owns TMEM and one elected lane issues tcgen05.mma,
// releasing each stage with tcgen05.commit onto an mbarrier. The operand loaders are the same
// im2col / transposed-view functors as the FFMA path, so every conv kind runs on this kernel.
namespace tc {

constexpr int BM = 128, BK = 16, NPROD = 256, NTHR = 288;   // 8 producer warps + 1 MMA warp

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t a, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t a) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ bool mbar_try(uint32_t a, uint32_t parity) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
               : "=r"(ok) : "r"(a), "r"(parity) : "memory");
  return ok != 0;
}
__device__ __forceinline__ bool mbar_test(uint32_t a, uint32_t parity) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
               : "=r"(ok) : "r"(a), "r"(parity) : "memory");
  return ok != 0;
}
#ifndef ORION_MBAR_SPIN
#define ORION_MBAR_SPIN 0
#endif
__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t parity) {
  if (ORION_MBAR_SPIN) { while (!mbar_test(a, parity)) {} }
  else { while (!mbar_try(a, parity)) {} }
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const float* src) {
  // zero-fill when src == nullptr (src-size 0 reads nothing; the address operand must still be valid)
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src ? src : reinterpret_cast<const float*>(&cp_async16)),
               "r"(src ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp_async4(uint32_t dst, const float* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(dst), "l"(src ? src : reinterpret_cast<const float*>(&cp_async16)),
               "r"(src ? 4 : 0) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N_>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N_) : "memory"); }
__device__ __forceinline__ float tf32_rna(float x) {
  uint32_t u;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(u) : "f"(x));
  return __uint_as_float(u);
}
// UMMA shared-memory descriptor, K-major, no swizzle: LBO = byte stride between the two 16-byte
// K halves of an 8x(32 B) core-matrix pair, SBO = byte stride between 8-row groups; version 1.
__device__ __forceinline__ uint64_t sdesc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) |
         (1ull << 46);
}
__device__ __forceinline__ void mma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}"
               ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t mbar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(mbar) : "memory");
}
// 32 consecutive TMEM columns of this thread's lane; tmem_ld32_nw leaves the wait to the caller
// (tmem_wait_ld) so several loads can be in flight.
#define TMEM_LD32_ASM(taddr, r)                                                                                   \
  asm volatile(                                                                                                 \
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"           \
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"                                \
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), \
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),    \
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),   \
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])                 \
      : "r"(taddr))
__device__ __forceinline__ void tmem_ld32_nw(uint32_t taddr, uint32_t* r) { TMEM_LD32_ASM(taddr, r); }
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
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
struct TcCfg {
  static constexpr int STAGES = BN >= 128 ? 6 : 8;   // ~192 KB of stages: deep enough to cover L2/HBM latency
  static constexpr int A_BYTES = BM * BK * 4;   // one of hi / lo
  static constexpr int B_BYTES = BN * BK * 4;
  static constexpr int STAGE_BYTES = 2 * (A_BYTES + B_BYTES);
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 256;
  // three fp32 accumulators of BN columns: hi*hi for even / odd k-steps, and the two correction
  // products. The tensor core's fp32 accumulation truncates, so each chain's bias grows with its
  // length; splitting the chains keeps the GEMM within ~1e-6 of fp64.
  static constexpr int ACC_COLS = 3 * BN;
  static constexpr int TMEM_COLS = ACC_COLS <= 32 ? 32 : ACC_COLS <= 64 ? 64 : ACC_COLS <= 128 ? 128 : ACC_COLS <= 256 ? 256 : 512;
  // instruction descriptor: D f32 (bits 4-5 = 1), A/B tf32 (2 at bits 7-9 / 10-12), K-major A/B,
  // N>>3 at bits 17-22, M>>4 at bits 24-28
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
};

// Byte offset of the 4 consecutive k (quad kq of the 32-k tile) of operand row `row` in a stage
// buffer of `rows` rows: k-chunk j = kq/2 (one MMA K-step of 8 tf32, rows x 32 B), then the
// core-matrix layout ((8 rows, row groups), 2 halves): row group stride SBO = 256 B, half stride
// LBO = 128 B, row stride 16 B inside a core matrix.
__device__ __forceinline__ uint32_t elem_off(int row, int kq, int rows) {
  return (uint32_t)((kq >> 1) * (rows * 32) + (row >> 3) * 256 + (kq & 1) * 128 + (row & 7) * 16);
}

template <int BN, class LA, class LB>
__global__ void __launch_bounds__(NTHR, 1) gemm_tc_kernel(GemmParams p, LA la, LB lb, OrionSig sig) {
  using Cfg = TcCfg<BN>;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  // offset the shared array itself (not a uintptr_t round trip), so accesses stay LDS/STS
  unsigned char* smem = smem_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + Cfg::STAGES * Cfg::STAGE_BYTES);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * Cfg::STAGES + 1);
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + Cfg::STAGES), done_bar = smem_u32(bars + 2 * Cfg::STAGES);
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
  const int kbeg = blockIdx.z * p.kps;
  const int kend = min(p.K, kbeg + p.kps);
  const int nk = kend > kbeg ? (kend - kbeg + BK - 1) / BK : 0;

  if (tid == 0) {
    for (int s = 0; s < Cfg::STAGES; s++) { mbar_init(full0 + 8 * s, NPROD); mbar_init(empty0 + 8 * s, 1); }
    mbar_init(done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == NPROD / 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(Cfg::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp < NPROD / 32) {
    // ---------------- producers. Each thread owns fixed k-quads of one A row and one B row per
    // stage. Raw fp32 quads are copied global -> shared with cp.async (STAGES-1 stages in flight,
    // zero-fill for padding / out-of-range), then each thread splits its own quads in place
    // (hi = rna_tf32(x) over the raw copy, lo = x - hi into the lo buffer) and arrives on the
    // stage's full barrier after a proxy fence.
    constexpr int S = Cfg::STAGES;
    constexpr int KQ = BK / 4;                                    // k-quads per row per stage
    constexpr int A_TPR = NPROD / BM, A_QPT = KQ / A_TPR;          // 2 threads per A row
    constexpr int BROWS = BN < NPROD ? BN : NPROD;
    constexpr int B_TPR = NPROD / BROWS;
    constexpr int B_QPT = KQ / B_TPR >= 1 ? KQ / B_TPR : 1;
    const int a_row = tid % BM, a_q0 = (tid / BM) * A_QPT;
    typename LA::Row arow = la.row(m0 + a_row, p.M);
    const int b_row = tid % BROWS, b_q0 = (tid / BROWS) * B_QPT;
    const bool b_on = tid < B_TPR * BROWS && b_row < BN;
    typename LB::Col bcol = lb.col(n0 + b_row, p.N);
    auto issue = [&](int kt) {
      const int s = kt % S;
      const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
      const uint32_t a_hi = st, b_hi = st + 2 * Cfg::A_BYTES;
      const int k0 = kbeg + kt * BK;
      const auto ta = la.tile(k0, kend, BK);
      const auto tb = lb.tile(k0, kend, BK);
#pragma unroll
      for (int q = 0; q < A_QPT; q++) {
        const int k = k0 + (a_q0 + q) * 4;
        const uint32_t dst = a_hi + elem_off(a_row, a_q0 + q, BM);
        const float* src;
        if (la.quad(arow, ta, a_q0 + q, kend, src)) cp_async16(dst, src);
        else {
#pragma unroll
          for (int e = 0; e < 4; e++) cp_async4(dst + 4 * e, la.addr(arow, k + e, kend));
        }
      }
      if (b_on) {
#pragma unroll
        for (int q = 0; q < B_QPT; q++) {
          const int k = k0 + (b_q0 + q) * 4;
          const uint32_t dst = b_hi + elem_off(b_row, b_q0 + q, BN);
          const float* src;
          if (lb.quad(bcol, tb, b_q0 + q, kend, src)) cp_async16(dst, src);
          else {
#pragma unroll
            for (int e = 0; e < 4; e++) cp_async4(dst + 4 * e, lb.addr(bcol, k + e, kend));
          }
        }
      }
    };
    auto split = [](unsigned char* hi, unsigned char* lo, uint32_t off) {
      float4 v = *reinterpret_cast<float4*>(hi + off), h, l;
      h.x = tf32_rna(v.x); h.y = tf32_rna(v.y); h.z = tf32_rna(v.z); h.w = tf32_rna(v.w);
      l.x = v.x - h.x; l.y = v.y - h.y; l.z = v.z - h.z; l.w = v.w - h.w;
      *reinterpret_cast<float4*>(hi + off) = h;
      *reinterpret_cast<float4*>(lo + off) = l;
    };
    // prologue: stages 0 .. L-1 with L = S-2 loads in flight ahead of the stage being split; a refill
    // targets the stage the MMA released two steps earlier (never the one just handed to it)
    constexpr int L = S - 2;
#pragma unroll 1
    for (int kt = 0; kt < L; kt++) {
      if (kt < nk) issue(kt);
      cp_commit();
    }
#pragma unroll 1
    for (int kt = 0; kt < nk; kt++) {
      const int nxt = kt + L;
      if (nxt < nk) {
        if (nxt >= S) mbar_wait(empty0 + 8 * (nxt % S), ((uint32_t)(nxt / S) & 1u) ^ 1u);
        issue(nxt);
      }
      cp_commit();
      cp_wait<L>();                                      // this thread's copies for stage kt landed
      const int s = kt % S;
      unsigned char* st = smem + s * Cfg::STAGE_BYTES;
#pragma unroll
      for (int q = 0; q < A_QPT; q++) split(st, st + Cfg::A_BYTES, elem_off(a_row, a_q0 + q, BM));
      if (b_on) {
#pragma unroll
        for (int q = 0; q < B_QPT; q++)
          split(st + 2 * Cfg::A_BYTES, st + 2 * Cfg::A_BYTES + Cfg::B_BYTES, elem_off(b_row, b_q0 + q, BN));
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic-proxy writes -> tensor core
      mbar_arrive(full0 + 8 * s);
    }
  } else if (warp == NPROD / 32 && lane == 0) {
    // ---------------- MMA issuer (one thread)
    for (int kt = 0; kt < nk; kt++) {
      const int s = kt % Cfg::STAGES;
      const uint32_t ph = (uint32_t)(kt / Cfg::STAGES) & 1u;
      mbar_wait(full0 + 8 * s, ph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t st = smem_u32(smem + s * Cfg::STAGE_BYTES);
      const uint32_t a_hi = st, a_lo = st + Cfg::A_BYTES, b_hi = st + 2 * Cfg::A_BYTES, b_lo = b_hi + Cfg::B_BYTES;
#pragma unroll
      for (int j = 0; j < BK / 8; j++) {
        const uint64_t dah = sdesc(a_hi + j * BM * 32, 128, 256), dal = sdesc(a_lo + j * BM * 32, 128, 256);
        const uint64_t dbh = sdesc(b_hi + j * BN * 32, 128, 256), dbl = sdesc(b_lo + j * BN * 32, 128, 256);
        const uint32_t d_main = tmem + (uint32_t)((j & 1) * BN), d_corr = tmem + (uint32_t)(2 * BN);
        mma_tf32(d_corr, dal, dbh, Cfg::IDESC, (kt | j) != 0);
        mma_tf32(d_corr, dah, dbl, Cfg::IDESC, 1);
        mma_tf32(d_main, dah, dbh, Cfg::IDESC, (kt | (j >> 1)) != 0);
      }
      mma_commit(empty0 + 8 * s);   // frees the stage once these MMAs have read it
    }
    mma_commit(done_bar);           // accumulator complete
  }

  // ---------------- epilogue: TMEM -> registers -> shared tile -> coalesced global (or split partials)
  // The stage buffers are free once the accumulator is complete; the 128 epilogue threads (TMEM
  // lanes 0..127 = tile rows) park their rows in a padded shared tile, then write it out row-major
  // with 128-bit stores (consecutive threads on consecutive columns).
  if (warp < 4) {
    mbar_wait(done_bar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    constexpr int TS = BN + 4;   // padded row stride (floats): conflict-free 128-bit row writes
    float* tile = reinterpret_cast<float*>(smem);
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      float v[32];
      if (nk > 0) {
        const uint32_t lane_base = tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)c0;
        float e[32], o[32];
        tmem_ld32(lane_base, e);
        tmem_ld32(lane_base + BN, o);
        tmem_ld32(lane_base + 2 * BN, v);
#pragma unroll
        for (int i = 0; i < 32; i++) v[i] = (e[i] + o[i]) + v[i];
      } else {
#pragma unroll
        for (int i = 0; i < 32; i++) v[i] = 0.f;
      }
#pragma unroll
      for (int i = 0; i < 32; i += 4)
        *reinterpret_cast<float4*>(tile + tid * TS + c0 + i) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
    }
    asm volatile("bar.sync 1, 128;" ::: "memory");   // epilogue warps only
    float* base = p.split == 1 ? p.C : p.ws + (long long)blockIdx.z * p.M * p.N;
    const long long ld = p.split == 1 ? p.ldc : p.N;
    const bool vec = ((ld & 3) == 0) && ((n0 & 3) == 0) && ((reinterpret_cast<uintptr_t>(base) & 15) == 0) &&
                     (p.split > 1 || p.bias == nullptr);
    constexpr int QPR = BN / 4;   // float4 per tile row
    for (int e = tid; e < BM * QPR; e += 128) {
      const int r = e / QPR, c = (e % QPR) * 4;
      const int m = m0 + r, n = n0 + c;
      if (m >= p.M) continue;
      const float4 t4 = *reinterpret_cast<const float4*>(tile + r * TS + c);
      float* dst = base + (long long)m * ld + n;
      if (vec && n + 3 < p.N) {
        *reinterpret_cast<float4*>(dst) = t4;
      } else {
        const float tv[4] = {t4.x, t4.y, t4.z, t4.w};
#pragma unroll
        for (int i = 0; i < 4; i++)
          if (n + i < p.N) dst[i] = p.split == 1 ? tv[i] + (p.bias ? __ldg(p.bias + n + i) : 0.f) : tv[i];
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  if (p.split > 1) {
    split_finish(p, blockIdx.y * gridDim.x + blockIdx.x, m0, n0, BM, BN);
  } else {
    __syncthreads();
  }
  if (warp == NPROD / 32) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS) : "memory");
  }
  orion_signal(sig);
}

}  // namespace tc

// ---------------------------------------------------------------- multi-tile tcgen05 kernel
// Streaming GEMMs (M >> 128 with modest K and N: MobileNetV2's 1x1 convs and their data gradients
// at batch 96, ResNet's 1x1 convs) are HBM-bound, and a one-tile CTA spends most of its life in
// setup, pipeline fill and a serial epilogue. Here a CTA owns TPC consecutive output tiles (a
// shape-only count) with two TMEM accumulator buffers, so the epilogue of tile i (dedicated warps
// 0-3: TMEM -> registers -> per-warp padded staging -> coalesced 128-bit stores) runs while the
// producers (warps 4-11: cp.async -> in-place 3xTF32 hi/lo split) and the MMA thread (warp 12) work
// on tile i+1, with 6-8 operand stages in flight. A CTA lives for TPC tiles only: no whole-GPU persistent grid,
// so an HP kernel's CTAs find a free SM within a few microseconds (kernels are not preemptible,
// P:670-689). Each tile is computed by one CTA in fixed k order: results do not depend on which
// CTA or SM runs it. Accumulators: one chain for hi*hi, one for the two correction products.
namespace tcm {
using namespace tc;
constexpr int BM = 128, BK = 16, NPROD = 256, NTHR = 416;   // 4 epilogue + 8 producer + 1 MMA warps
constexpr int MMA_WARP = 4 + NPROD / 32;
constexpr int EPI_LD = 36;                                   // padded staging row (floats): conflict-free
constexpr int EPI_BYTES = 4 * 32 * EPI_LD * 4;
// BN = 64 or 128 output columns per tile; one CTA per SM with STAGES deep enough to keep ~80 KB of
// operand loads in flight per SM (an HBM-bound stream needs latency x bandwidth / #SM bytes).
template <int BN_>
struct Cfg {
  static constexpr int BN = BN_;
  static constexpr int A_BYTES = BM * BK * 4, B_BYTES = BN * BK * 4, STAGE_BYTES = 2 * (A_BYTES + B_BYTES);
  // RAW_STAGES landing slots (raw fp32, cp.async) feed STAGES split slots (hi/lo, read by the MMA):
  // ~100 KB of loads in flight per SM for HBM-bound streams.
  static constexpr int RAW_BYTES = A_BYTES + B_BYTES;
  static constexpr int RAW_STAGES = BN == 64 ? 10 : 8, STAGES = BN == 64 ? 3 : 2;
  static constexpr int SMEM = RAW_STAGES * RAW_BYTES + STAGES * STAGE_BYTES + EPI_BYTES + 256 + 1024;
  static constexpr int TMEM_COLS = 4 * BN;                   // 2 buffers x (main, corr)
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
};

struct Params { int M, N, K; float* C; long long ldc; const float* bias; int tiles_n, tiles, tpc, dbg; };

template <int BN_, class LA, class LB>
__global__ void __launch_bounds__(NTHR, 1) gemm_tcm_kernel(Params p, LA la, LB lb, OrionSig sig) {
  using C_ = Cfg<BN_>;
  constexpr int BN = C_::BN, A_BYTES = C_::A_BYTES, B_BYTES = C_::B_BYTES, STAGE_BYTES = C_::STAGE_BYTES, STAGES = C_::STAGES;
  constexpr int RAW_BYTES = C_::RAW_BYTES, RAW_STAGES = C_::RAW_STAGES;
  constexpr int TMEM_COLS = C_::TMEM_COLS;
  constexpr uint32_t IDESC = C_::IDESC;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  // offset the shared array itself (not a uintptr_t round trip), so accesses stay LDS/STS
  unsigned char* smem = smem_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_raw) & 1023u)) & 1023u);
  unsigned char* raw = smem + STAGES * STAGE_BYTES;
  float* epi = reinterpret_cast<float*>(raw + RAW_STAGES * RAW_BYTES);
  uint64_t* bars = reinterpret_cast<uint64_t*>(raw + RAW_STAGES * RAW_BYTES + EPI_BYTES);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * STAGES + 4);
  const uint32_t full0 = smem_u32(bars), empty0 = full0 + 8 * STAGES, tfull0 = empty0 + 8 * STAGES, tempty0 = tfull0 + 16;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int t0 = blockIdx.x * p.tpc;
  const int ntl = min(p.tpc, p.tiles - t0);
  const int nk = (p.K + BK - 1) / BK;
  const int G = ntl * nk;   // (tile, k-tile) steps of this CTA

  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) { mbar_init(full0 + 8 * s, NPROD); mbar_init(empty0 + 8 * s, 1); }
    for (int b = 0; b < 2; b++) { mbar_init(tfull0 + 8 * b, 1); mbar_init(tempty0 + 8 * b, 4); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "r"(TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp >= 4 && warp < MMA_WARP) {
    // ---------------- producers: thread pt stages the quads idx = pt + 128 j with row = 8 (idx / 32)
    // + idx % 8 and quad = (idx / 8) % 4: a warp instruction covers 8 rows x 4 quads (whole 64-byte
    // row pieces, coalesced), and the 8 threads of each shared-memory phase hit 8 rows of one core
    // matrix column (16 B apart in the K-major layout): conflict-free.
    const int pt = tid - 128;
    auto row_of = [](int idx) { return ((idx >> 5) << 3) | (idx & 7); };
    auto quad_of = [](int idx) { return (idx >> 3) & 3; };
    auto issue = [&](int g) {
      const int t = t0 + g / nk, kt = g % nk;
      const int m0 = (t / p.tiles_n) * BM, n0 = (t % p.tiles_n) * BN;
      const uint32_t st = smem_u32(raw + (g % RAW_STAGES) * RAW_BYTES);
      const uint32_t a_hi = st, b_hi = st + A_BYTES;
      const int k0 = kt * BK;
      const auto ta = la.tile(k0, p.K, BK);
      const auto tb = lb.tile(k0, p.K, BK);
#pragma unroll
      for (int j = 0; j < BM * 4 / NPROD; j++) {
        const int idx = pt + NPROD * j, row = row_of(idx), q = quad_of(idx);
        const typename LA::Row ar = la.row(m0 + row, p.M);
        const uint32_t dst = a_hi + elem_off(row, q, BM);
        const float* src;
        if (la.quad(ar, ta, q, p.K, src)) cp_async16(dst, src);
        else {
#pragma unroll
          for (int e = 0; e < 4; e++) cp_async4(dst + 4 * e, la.addr(ar, k0 + 4 * q + e, p.K));
        }
      }
#pragma unroll
      for (int j = 0; j < BN * 4 / NPROD; j++) {
        const int idx = pt + NPROD * j, row = row_of(idx), q = quad_of(idx);
        const typename LB::Col bc = lb.col(n0 + row, p.N);
        const uint32_t dst = b_hi + elem_off(row, q, BN);
        const float* src;
        if (lb.quad(bc, tb, q, p.K, src)) cp_async16(dst, src);
        else {
#pragma unroll
          for (int e = 0; e < 4; e++) cp_async4(dst + 4 * e, lb.addr(bc, k0 + 4 * q + e, p.K));
        }
      }
    };
    auto split = [](const unsigned char* src, unsigned char* hi, unsigned char* lo, uint32_t off) {
      float4 v = *reinterpret_cast<const float4*>(src + off), h, l;
      h.x = tf32_rna(v.x); h.y = tf32_rna(v.y); h.z = tf32_rna(v.z); h.w = tf32_rna(v.w);
      l.x = v.x - h.x; l.y = v.y - h.y; l.z = v.z - h.z; l.w = v.w - h.w;
      *reinterpret_cast<float4*>(hi + off) = h;
      *reinterpret_cast<float4*>(lo + off) = l;
    };
    // Each thread splits exactly the quads it copied, so a raw slot is free for this thread's next
    // copy as soon as its own split of that slot is done (program order): L = RAW_STAGES - 1 steps of
    // loads in flight without any cross-thread wait; only the split slots wait for the MMA.
    constexpr int L = RAW_STAGES - 1;
#pragma unroll 1
    for (int g = 0; g < L; g++) {
      if (g < G) issue(g);
      cp_commit();
    }
#pragma unroll 1
    for (int g = 0; g < G; g++) {
      if (g + L < G && !(p.dbg & 2)) issue(g + L);
      cp_commit();
      cp_wait<L>();                                   // this thread's copies for step g landed
      const int s = g % STAGES;
      if (g >= STAGES) mbar_wait(empty0 + 8 * s, ((uint32_t)(g / STAGES) & 1u) ^ 1u);   // MMA released slot s
      const unsigned char* rw = raw + (g % RAW_STAGES) * RAW_BYTES;
      unsigned char* st = smem + s * STAGE_BYTES;
#pragma unroll
      for (int j = 0; j < BM * 4 / NPROD; j++) {
        const int idx = pt + NPROD * j;
        split(rw, st, st + A_BYTES, elem_off(row_of(idx), quad_of(idx), BM));
      }
#pragma unroll
      for (int j = 0; j < BN * 4 / NPROD; j++) {
        const int idx = pt + NPROD * j;
        split(rw + A_BYTES, st + 2 * A_BYTES, st + 2 * A_BYTES + B_BYTES, elem_off(row_of(idx), quad_of(idx), BN));
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive(full0 + 8 * s);
    }
  } else if (warp == MMA_WARP && lane == 0) {
    // ---------------- MMA issuer
#pragma unroll 1
    for (int g = 0; g < G; g++) {
      const int i = g / nk, kt = g % nk, buf = i & 1;
      if (kt == 0) {
        mbar_wait(tempty0 + 8 * buf, ((uint32_t)(i >> 1) & 1u) ^ 1u);   // epilogue drained this buffer
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      }
      const int s = g % STAGES;
      mbar_wait(full0 + 8 * s, (uint32_t)(g / STAGES) & 1u);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t st = smem_u32(smem + s * STAGE_BYTES);
      const uint32_t a_hi = st, a_lo = st + A_BYTES, b_hi = st + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
      const uint32_t d_main = tmem + (uint32_t)(buf * 2 * BN), d_corr = d_main + BN;
#pragma unroll
      for (int j = 0; j < BK / 8; j++) {
        const uint64_t dah = sdesc(a_hi + j * BM * 32, 128, 256), dal = sdesc(a_lo + j * BM * 32, 128, 256);
        const uint64_t dbh = sdesc(b_hi + j * BN * 32, 128, 256), dbl = sdesc(b_lo + j * BN * 32, 128, 256);
        mma_tf32(d_corr, dal, dbh, IDESC, (kt | j) != 0);
        mma_tf32(d_corr, dah, dbl, IDESC, 1);
        mma_tf32(d_main, dah, dbh, IDESC, (kt | j) != 0);
      }
      mma_commit(empty0 + 8 * s);
      if (kt == nk - 1) mma_commit(tfull0 + 8 * buf);
    }
  } else if (warp < 4) {
    // ---------------- epilogue: warp w owns tile rows 32w..32w+31 (TMEM lanes)
    float* stg = epi + warp * 32 * EPI_LD;
    const bool vec = ((p.ldc & 3) == 0) && ((reinterpret_cast<uintptr_t>(p.C) & 15) == 0);
    const int rr = lane >> 3, cq = (lane & 7) * 4;
#pragma unroll 1
    for (int i = 0; i < ntl; i++) {
      const int buf = i & 1, t = t0 + i;
      const int m0 = (t / p.tiles_n) * BM, n0 = (t % p.tiles_n) * BN;
      mbar_wait(tfull0 + 8 * buf, (uint32_t)(i >> 1) & 1u);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll 1
      for (int c0 = 0; c0 < BN && n0 + c0 < p.N && !(p.dbg & 4); c0 += 32) {
        uint32_t mv[32], cv[32];
        const uint32_t base = tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)(buf * 2 * BN + c0);
        tmem_ld32_nw(base, mv);
        tmem_ld32_nw(base + BN, cv);
        tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < 32; j += 4)
          *reinterpret_cast<float4*>(stg + lane * EPI_LD + j) =
              make_float4(__uint_as_float(mv[j]) + __uint_as_float(cv[j]), __uint_as_float(mv[j + 1]) + __uint_as_float(cv[j + 1]),
                          __uint_as_float(mv[j + 2]) + __uint_as_float(cv[j + 2]), __uint_as_float(mv[j + 3]) + __uint_as_float(cv[j + 3]));
        __syncwarp();
        // all 8 staged rows into distinct registers first, then the 8 stores: a store's source
        // registers are not recycled by the next load (no serialisation on store data read-out)
        float4 vv[8];
#pragma unroll
        for (int it = 0; it < 8; it++) vv[it] = *reinterpret_cast<const float4*>(stg + (it * 4 + rr) * EPI_LD + cq);
#pragma unroll
        for (int it = 0; it < 8; it++) {
          const int r = it * 4 + rr;
          const int m = m0 + 32 * warp + r, n = n0 + c0 + cq;
          if (m < p.M && n < p.N && !(p.dbg & 1)) {
            float4 v = vv[it];
            float* dst = p.C + (long long)m * p.ldc + n;
            if (vec && n + 3 < p.N) {
              if (p.bias) { v.x += __ldg(p.bias + n); v.y += __ldg(p.bias + n + 1); v.z += __ldg(p.bias + n + 2); v.w += __ldg(p.bias + n + 3); }
              *reinterpret_cast<float4*>(dst) = v;
            } else {
              const float tv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
              for (int e = 0; e < 4; e++)
                if (n + e < p.N) dst[e] = tv[e] + (p.bias ? __ldg(p.bias + n + e) : 0.f);
            }
          }
        }
        __syncwarp();
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty0 + 8 * buf);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
  }
  orion_signal(sig);
}

// Shape-only plan: the kernel takes streaming shapes with enough tiles to fill the part's 148 SMs
// without a K split; BN = 128 when N > 64 (A read once for N <= 128); a CTA's tile count targets
// ~4 waves (<= 16 tiles, so a CTA lives a few microseconds).
inline int bn_for(long long N) { return N > 64 ? 128 : 64; }
inline long long tiles_of(long long M, long long N) { return cdiv(M, BM) * cdiv(N, bn_for(N)); }
inline bool ok(long long M, long long N, long long K) { return K >= 8 && K <= 2048 && tiles_of(M, N) >= 2 * 148; }
inline int tpc_of(long long tiles) {
  long long t = cdiv(tiles, 148 * 4);
  return (int)(t < 1 ? 1 : t > 16 ? 16 : t);
}
template <int BN, class LA, class LB>
bool prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  bool okk = cudaFuncSetAttribute((const void*)gemm_tcm_kernel<BN, LA, LB>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::SMEM) ==
             cudaSuccess;
  if (okk) done.store(1, std::memory_order_release);
  return okk;
}
template <class LA, class LB>
void geom(LaunchGeom* g, long long M, long long N) {
  const long long tiles = tiles_of(M, N);
  g->grid = dim3((unsigned)cdiv(tiles, tpc_of(tiles))); g->block = dim3(NTHR);
  if (bn_for(N) == 128) { prepare<128, LA, LB>(); g->smem = Cfg<128>::SMEM; g->func = (const void*)gemm_tcm_kernel<128, LA, LB>; }
  else { prepare<64, LA, LB>(); g->smem = Cfg<64>::SMEM; g->func = (const void*)gemm_tcm_kernel<64, LA, LB>; }
  g->pipe = ORION_PIPE_TF32X3;
}
template <class LA, class LB>
bool is(const void* f) { return f == (const void*)gemm_tcm_kernel<128, LA, LB> || f == (const void*)gemm_tcm_kernel<64, LA, LB>; }
template <class LA, class LB>
int launch(const LaunchGeom& g, long long M, long long N, long long K, float* C, long long ldc, const float* bias, LA la, LB lb,
           OrionSig sig, cudaStream_t s) {
  Params p;
  p.M = (int)M; p.N = (int)N; p.K = (int)K; p.C = C; p.ldc = ldc; p.bias = bias;
  p.tiles_n = (int)cdiv(N, bn_for(N)); p.tiles = (int)tiles_of(M, N); p.tpc = tpc_of(p.tiles);
  static const int dbg = getenv("ORION_TCM_DEBUG") ? atoi(getenv("ORION_TCM_DEBUG")) : 0;   // 1 no stores, 2 no loads, 4 no epilogue
  p.dbg = dbg;
  if (bn_for(N) == 128) {
    if (!prepare<128, LA, LB>()) return ORION_E_CUDA;
    gemm_tcm_kernel<128, LA, LB><<<g.grid, g.block, g.smem, s>>>(p, la, lb, sig);
  } else {
    if (!prepare<64, LA, LB>()) return ORION_E_CUDA;
    gemm_tcm_kernel<64, LA, LB><<<g.grid, g.block, g.smem, s>>>(p, la, lb, sig);
  }
  return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
}
}  // namespace tcm

// ---------------------------------------------------------------- TMA-fed multi-tile tcgen05 kernel
// The dense streaming case (row-major A with K % 4 == 0: 1x1-conv forward and data gradient), fed
// and drained by the Tensor Memory Accelerator. A 2-D tensor map with 128-byte swizzle lands a
// BM x 32 tile directly in the UMMA K-major SWIZZLE_128B layout, so the raw fp32 tile IS the "hi"
// operand: the tensor core reads tf32 by truncating the low 13 mantissa bits (measured,
// tools/probe/tma_tf32.cu). Converter warps only form lo = x - trunc_tf32(x) (exact in fp32) at
// the same offsets; D += A_lo B_hi + A_hi B_lo + A_hi B_hi (dropped A_lo B_lo < 2^-20 |ab|). B given
// [K][N] (data gradient: W) lands as [32][BN] and the converters transpose it into the K-major
// layout (hi and lo). The epilogue stages 32 x 32 blocks in 128B-swizzled shared memory (conflict
// free) and stores them with TMA (double-buffered per warp), so no thread waits on global stores.
// Roles: warps 0-3 epilogue (TMEM lanes), 4-7 converters, warp 8 lane 0 TMA producer, warp 9 lane 0
// MMA issuer and TMEM owner. Each tile is computed by one CTA in fixed k order (deterministic).
namespace tmk {
using namespace tc;
constexpr int BM = 128, BK = 32, NCONV = 128, NTHR = 320, CONV_WARPS = NCONV / 32;
constexpr int TMA_WARP = 4 + CONV_WARPS, MMA_WARP = TMA_WARP + 1;
constexpr int EPI_BUF = 32 * 32 * 4, EPI_BYTES = 4 * 2 * EPI_BUF;   // per warp: 2 staging blocks of 32 x 32
template <int BN_, bool BMN_>
struct Cfg {
  static constexpr int BN = BN_;
  static constexpr int A_BYTES = BM * BK * 4, B_BYTES = BN * BK * 4;
  // stage: [A hi (TMA)][A lo][B hi][B lo][B raw (MN-major B only)]
  static constexpr int STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES + (BMN_ ? B_BYTES : 0);
  static constexpr int STAGES = (194 * 1024) / STAGE_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + EPI_BYTES + 256 + 1024;
  static constexpr int TMEM_COLS = 4 * BN;
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
  static constexpr uint32_t TX_BYTES = A_BYTES + B_BYTES;
};
struct Params { int M, N, K; const float* bias; int tiles_n, tiles, tpc; };

__device__ __forceinline__ void tma2d(uint32_t dst, const CUtensorMap* tm, int c0, int c1, uint32_t bar) {
  asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst), "l"(tm),
               "r"(c0), "r"(c1), "r"(bar) : "memory");
}
__device__ __forceinline__ void tma2d_store(const CUtensorMap* tm, int c0, int c1, uint32_t src) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(tm), "r"(c0), "r"(c1), "r"(src) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ float trunc_tf32(float x) { return __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); }
__device__ __forceinline__ float4 lo4(const float4 v) {
  return make_float4(v.x - trunc_tf32(v.x), v.y - trunc_tf32(v.y), v.z - trunc_tf32(v.z), v.w - trunc_tf32(v.w));
}
// UMMA descriptor, K-major SWIZZLE_128B: 8-row atoms of 128-byte rows (32 tf32), SBO = 1024 B between
// atoms, LBO unused; layout type 2 at bits 61-63; k-step j advances the start address by 32 B.
__device__ __forceinline__ uint64_t sdesc128(uint32_t addr) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | (1ull << 16) | ((uint64_t)(1024 >> 4) << 32) | (1ull << 46) | (2ull << 61);
}
// byte offset of element (row, col < 32) of a 32-float-wide SWIZZLE_128B tile (what TMA writes / reads)
__device__ __forceinline__ uint32_t sw128_off(int row, int col) {
  return (uint32_t)((row >> 3) * 1024 + (row & 7) * 128 + (((col >> 2) ^ (row & 7)) << 4) + (col & 3) * 4);
}

template <int BN_, bool BMN>
__global__ void __launch_bounds__(NTHR, 1) gemm_tmk_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                                                          const __grid_constant__ CUtensorMap tmC, Params p, OrionSig sig) {
  using C_ = Cfg<BN_, BMN>;
  constexpr int BN = C_::BN, A_BYTES = C_::A_BYTES, B_BYTES = C_::B_BYTES, STAGE_BYTES = C_::STAGE_BYTES, STAGES = C_::STAGES;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  // offset the shared array itself (not a uintptr_t round trip), so accesses stay LDS/STS
  unsigned char* smem = smem_raw + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_raw) & 1023u)) & 1023u);
  unsigned char* epi = smem + STAGES * STAGE_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(epi + EPI_BYTES);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 * STAGES + 4);
  const uint32_t tfull0 = smem_u32(bars), cfull0 = tfull0 + 8 * STAGES, empty0 = cfull0 + 8 * STAGES;
  const uint32_t afull0 = empty0 + 8 * STAGES, aempty0 = afull0 + 16;   // TMEM accumulator buffers
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int t0 = blockIdx.x * p.tpc;
  const int ntl = min(p.tpc, p.tiles - t0);
  const int nk = (p.K + BK - 1) / BK;
  const int G = ntl * nk;

  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) { mbar_init(tfull0 + 8 * s, 1); mbar_init(cfull0 + 8 * s, CONV_WARPS); mbar_init(empty0 + 8 * s, 1); }
    for (int b = 0; b < 2; b++) { mbar_init(afull0 + 8 * b, 1); mbar_init(aempty0 + 8 * b, 4); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == TMA_WARP && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
  }
  if (warp == 0 && lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmC) : "memory");
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
#pragma unroll 1
      for (int g = 0; g < G; g++) {
        const int s = g % STAGES;
        if (g >= STAGES) mbar_wait(empty0 + 8 * s, ((uint32_t)(g / STAGES) & 1u) ^ 1u);
        const int t = t0 + g / nk, kt = g % nk;
        const int m0 = (t / p.tiles_n) * BM, n0 = (t % p.tiles_n) * BN;
        const uint32_t st = smem_u32(smem + s * STAGE_BYTES), bar = tfull0 + 8 * s;
        mbar_expect(bar, C_::TX_BYTES);
        tma2d(st, &tmA, kt * BK, m0, bar);
        if (BMN) tma2d(st + 2 * A_BYTES + 2 * B_BYTES, &tmB, n0, kt * BK, bar);
        else tma2d(st + 2 * A_BYTES, &tmB, kt * BK, n0, bar);
      }
    }
  } else if (warp >= 4 && warp < TMA_WARP) {
    // ---------------- converters: lo = x - trunc(x) for A (and B); B transposed when MN-major
    const int ct = tid - 128;
#pragma unroll 1
    for (int g = 0; g < G; g++) {
      const int s = g % STAGES;
      mbar_wait(tfull0 + 8 * s, (uint32_t)(g / STAGES) & 1u);
      unsigned char* st = smem + s * STAGE_BYTES;
      const float4* ahi = reinterpret_cast<const float4*>(st);
      float4* alo = reinterpret_cast<float4*>(st + A_BYTES);
      constexpr int AQ = A_BYTES / 16 / NCONV;
      float4 va[AQ];
#pragma unroll
      for (int j = 0; j < AQ; j++) va[j] = ahi[ct + NCONV * j];
#pragma unroll
      for (int j = 0; j < AQ; j++) alo[ct + NCONV * j] = lo4(va[j]);
      constexpr int BQ = B_BYTES / 16 / NCONV;
      if (!BMN) {
        const float4* bhi = reinterpret_cast<const float4*>(st + 2 * A_BYTES);
        float4* blo = reinterpret_cast<float4*>(st + 2 * A_BYTES + B_BYTES);
        float4 vb[BQ];
#pragma unroll
        for (int j = 0; j < BQ; j++) vb[j] = bhi[ct + NCONV * j];
#pragma unroll
        for (int j = 0; j < BQ; j++) blo[ct + NCONV * j] = lo4(vb[j]);
      } else {
        // raw [32 k][BN n] -> K-major SWIZZLE_128B (n, k): thread item = (row n, k-quad kq); reads are
        // consecutive n across lanes, writes one 16-byte chunk per row (swizzle spreads 8 rows over 8 chunks)
        const float* braw = reinterpret_cast<const float*>(st + 2 * A_BYTES + 2 * B_BYTES);
        unsigned char* bhi = st + 2 * A_BYTES;
        unsigned char* blo = st + 2 * A_BYTES + B_BYTES;
#pragma unroll
        for (int j = 0; j < BQ; j++) {
          const int idx = ct + NCONV * j;
          const int n = idx % BN, kq = idx / BN;
          const float4 v = make_float4(braw[(4 * kq) * BN + n], braw[(4 * kq + 1) * BN + n], braw[(4 * kq + 2) * BN + n], braw[(4 * kq + 3) * BN + n]);
          const uint32_t off = sw128_off(n, 4 * kq);
          *reinterpret_cast<float4*>(bhi + off) = make_float4(trunc_tf32(v.x), trunc_tf32(v.y), trunc_tf32(v.z), trunc_tf32(v.w));
          *reinterpret_cast<float4*>(blo + off) = lo4(v);
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(cfull0 + 8 * s);
    }
  } else if (warp == MMA_WARP && lane == 0) {
#pragma unroll 1
    for (int g = 0; g < G; g++) {
      const int i = g / nk, kt = g % nk, buf = i & 1;
      if (kt == 0) {
        mbar_wait(aempty0 + 8 * buf, ((uint32_t)(i >> 1) & 1u) ^ 1u);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      }
      const int s = g % STAGES;
      mbar_wait(tfull0 + 8 * s, (uint32_t)(g / STAGES) & 1u);
      mbar_wait(cfull0 + 8 * s, (uint32_t)(g / STAGES) & 1u);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t st = smem_u32(smem + s * STAGE_BYTES);
      const uint32_t a_hi = st, a_lo = st + A_BYTES, b_hi = st + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
      const uint32_t d_main = tmem + (uint32_t)(buf * 2 * BN), d_corr = d_main + BN;
#pragma unroll
      for (int j = 0; j < BK / 8; j++) {
        const uint64_t dah = sdesc128(a_hi + 32 * j), dal = sdesc128(a_lo + 32 * j);
        const uint64_t dbh = sdesc128(b_hi + 32 * j), dbl = sdesc128(b_lo + 32 * j);
        mma_tf32(d_corr, dal, dbh, C_::IDESC, (kt | j) != 0);
        mma_tf32(d_corr, dah, dbl, C_::IDESC, 1);
        mma_tf32(d_main, dah, dbh, C_::IDESC, (kt | j) != 0);
      }
      mma_commit(empty0 + 8 * s);
      if (kt == nk - 1) mma_commit(afull0 + 8 * buf);
    }
  } else if (warp < 4) {
    // ---------------- epilogue: warp w owns tile rows 32w..32w+31 (TMEM lanes); per 32-column chunk:
    // TMEM -> registers (+ bias) -> swizzled staging block -> TMA store (lane 0), two blocks in flight
    unsigned char* stg0 = epi + warp * 2 * EPI_BUF;
    int nst = 0;   // stores issued by this warp
#pragma unroll 1
    for (int i = 0; i < ntl; i++) {
      const int buf = i & 1, t = t0 + i;
      const int m0 = (t / p.tiles_n) * BM, n0 = (t % p.tiles_n) * BN;
      mbar_wait(afull0 + 8 * buf, (uint32_t)(i >> 1) & 1u);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll 1
      for (int c0 = 0; c0 < BN && n0 + c0 < p.N; c0 += 32) {
        uint32_t mv[32], cv[32];
        const uint32_t base = tmem + ((uint32_t)(32 * warp) << 16) + (uint32_t)(buf * 2 * BN + c0);
        tmem_ld32_nw(base, mv);
        tmem_ld32_nw(base + BN, cv);
        unsigned char* stg = stg0 + (nst & 1) * EPI_BUF;
        if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");   // this block's previous store read it
        tmem_wait_ld();
        __syncwarp();
#pragma unroll
        for (int j = 0; j < 32; j += 4) {
          float4 v = make_float4(__uint_as_float(mv[j]) + __uint_as_float(cv[j]), __uint_as_float(mv[j + 1]) + __uint_as_float(cv[j + 1]),
                                 __uint_as_float(mv[j + 2]) + __uint_as_float(cv[j + 2]), __uint_as_float(mv[j + 3]) + __uint_as_float(cv[j + 3]));
          if (p.bias) {
            const int n = n0 + c0 + j;
            if (n < p.N) v.x += __ldg(p.bias + n);
            if (n + 1 < p.N) v.y += __ldg(p.bias + n + 1);
            if (n + 2 < p.N) v.z += __ldg(p.bias + n + 2);
            if (n + 3 < p.N) v.w += __ldg(p.bias + n + 3);
          }
          *reinterpret_cast<float4*>(stg + sw128_off(lane, j)) = v;
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) {
          tma2d_store(&tmC, n0 + c0, m0 + 32 * warp, smem_u32(stg));
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
        nst++;
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(aempty0 + 8 * buf);
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // all of this warp's stores complete
    __syncwarp();
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C_::TMEM_COLS) : "memory");
  }
  orion_signal(sig);
}

// cuTensorMapEncodeTiled, resolved through cudart at first use (the library does not link libcuda)
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
// 2-D fp32 map of a row-major [rows][ld] array with `inner` columns, box {box_inner, box_rows}
inline bool map2d(CUtensorMap* m, const float* base, long long rows, long long inner, long long ld, int box_inner, int box_rows,
                  CUtensorMapSwizzle sw) {
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
  cuuint32_t box[2] = {(cuuint32_t)box_inner, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  return encoder()(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
inline bool al16p(const void* q) { return (reinterpret_cast<uintptr_t>(q) & 15) == 0; }
// dense row-major A [M][lda] (K contiguous); B^T [N][ldb] (bmn = false) or B [K][ldb] (bmn = true); C [M][ldc]
inline bool ok(long long M, long long N, long long K, long long lda, long long ldb, long long ldc, const float* A, const float* B,
               const float* C) {
  return tcm::ok(M, N, K) && K % 4 == 0 && lda % 4 == 0 && ldb % 4 == 0 && ldc % 4 == 0 && al16p(A) && al16p(B) && al16p(C) &&
         encoder() != nullptr;
}
template <int BN, bool BMN>
bool prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  bool okk = cudaFuncSetAttribute((const void*)gemm_tmk_kernel<BN, BMN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN, BMN>::SMEM) ==
             cudaSuccess;
  if (okk) done.store(1, std::memory_order_release);
  return okk;
}
template <int BN, bool BMN>
void geom_t(LaunchGeom* g, long long tiles) {
  prepare<BN, BMN>();
  g->grid = dim3((unsigned)cdiv(tiles, tcm::tpc_of(tiles))); g->block = dim3(NTHR); g->smem = Cfg<BN, BMN>::SMEM;
  g->func = (const void*)gemm_tmk_kernel<BN, BMN>;
  g->pipe = ORION_PIPE_TF32X3;
}
inline void geom(LaunchGeom* g, long long M, long long N, bool bmn) {
  const long long tiles = tcm::tiles_of(M, N);
  if (tcm::bn_for(N) == 128) { if (bmn) geom_t<128, true>(g, tiles); else geom_t<128, false>(g, tiles); }
  else { if (bmn) geom_t<64, true>(g, tiles); else geom_t<64, false>(g, tiles); }
}
inline bool is(const void* f) {
  return f == (const void*)gemm_tmk_kernel<128, true> || f == (const void*)gemm_tmk_kernel<128, false> ||
         f == (const void*)gemm_tmk_kernel<64, true> || f == (const void*)gemm_tmk_kernel<64, false>;
}
template <int BN, bool BMN>
int launch_t(const LaunchGeom& g, const Params& p, const float* A, long long lda, const float* B, long long ldb, float* C, long long ldc,
             OrionSig sig, cudaStream_t s) {
  if (!prepare<BN, BMN>()) return ORION_E_CUDA;
  CUtensorMap ma, mb, mc;
  if (!map2d(&ma, A, p.M, p.K, lda, BK, BM, CU_TENSOR_MAP_SWIZZLE_128B)) return ORION_E_CUDA;
  if (BMN ? !map2d(&mb, B, p.K, p.N, ldb, BN, BK, CU_TENSOR_MAP_SWIZZLE_NONE) : !map2d(&mb, B, p.N, p.K, ldb, BK, BN, CU_TENSOR_MAP_SWIZZLE_128B))
    return ORION_E_CUDA;
  if (!map2d(&mc, C, p.M, p.N, ldc, 32, 32, CU_TENSOR_MAP_SWIZZLE_128B)) return ORION_E_CUDA;
  gemm_tmk_kernel<BN, BMN><<<g.grid, g.block, g.smem, s>>>(ma, mb, mc, p, sig);
  return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
}
inline int launch(const LaunchGeom& g, long long M, long long N, long long K, float* C, long long ldc, const float* bias, const float* A,
                  long long lda, const float* B, long long ldb, bool bmn, OrionSig sig, cudaStream_t s) {
  Params p;
  p.M = (int)M; p.N = (int)N; p.K = (int)K; p.bias = bias;
  p.tiles_n = (int)cdiv(N, tcm::bn_for(N)); p.tiles = (int)tcm::tiles_of(M, N); p.tpc = tcm::tpc_of(p.tiles);
  if (tcm::bn_for(N) == 128)
    return bmn ? launch_t<128, true>(g, p, A, lda, B, ldb, C, ldc, sig, s) : launch_t<128, false>(g, p, A, lda, B, ldb, C, ldc, sig, s);
  return bmn ? launch_t<64, true>(g, p, A, lda, B, ldb, C, ldc, sig, s) : launch_t<64, false>(g, p, A, lda, B, ldb, C, ldc, sig, s);
}
}  // namespace tmk


// ---------------------------------------------------------------- skinny A^T B (weight gradients)
// C[M][N] = sum_k A[k][m] B[k][n] for M, N <= 128 and very long K (1x1-conv weight gradients over
// N*H*W rows): HBM-bound, so the kernel streams 64-row blocks of both operands with coalesced
// 128-bit loads (the next block's loads in flight while the current one is multiplied), keeps both
// blocks in shared memory and gives each thread a 4x4 register block of C over a fixed subset of
// the rows (row groups combined in fixed order). K is split over CTAs (shape-only count) and the
// splits are summed in order (split_finish).
namespace atb {
constexpr int NTH = 256;

// Variant <TMB, TNB, R, MAXM, MAXN>: each thread owns a TMB x TNB register block of C; R rows of
// both operands are staged per step. MAXQ = float4s each thread stages per step.
template <int TMB, int TNB, int R, int MAXM, int MAXN>
struct V {
  static constexpr int MAXQ = (R * ((MAXM + MAXN) / 4) + NTH - 1) / NTH;
  __host__ __device__ static int pad_dim(int d) { return ((d + 3) / 4) * 4 + 4; }
  __host__ __device__ static int smem_bytes(int M, int N) { return (2 * R * (pad_dim(M) + pad_dim(N)) + NTH * TMB * TNB) * 4; }
  __host__ __device__ static bool fits(long long M, long long N) {
    return M <= MAXM && N <= MAXN && ((M + TMB - 1) / TMB) * ((N + TNB - 1) / TNB) <= NTH;
  }
};
using V44 = V<4, 4, 64, 128, 128>;
using V84 = V<8, 4, 32, 192, 64>;
using V48 = V<4, 8, 32, 64, 192>;

template <class VV, int TMB, int TNB, int R>
__global__ void __launch_bounds__(NTH) gemm_atb_kernel(GemmParams p, const float* __restrict__ A, long long lda,
                                                      const float* __restrict__ B, long long ldb, OrionSig sig) {
  extern __shared__ __align__(16) float atb_smem[];
  constexpr int MAXQ = VV::MAXQ;
  const int tid = threadIdx.x;
  const int M = p.M, N = p.N;
  const int Mp = VV::pad_dim(M), Np = VV::pad_dim(N);
  float* As0 = atb_smem;                  // [2][R][Mp]
  float* Bs0 = As0 + 2 * R * Mp;          // [2][R][Np]
  float* red = Bs0 + 2 * R * Np;          // [NTH * TMB * TNB]
  const int mb = (M + TMB - 1) / TMB, nb = (N + TNB - 1) / TNB;
  const int nblk = mb * nb;
  const int G = NTH / nblk;                            // row groups
  const int grp = tid / nblk, blk = tid % nblk;
  const int bm = (blk / nb) * TMB, bn = (blk % nb) * TNB;
  const bool active = grp < G;
  const int kbeg = blockIdx.z * p.kps;
  const int kend = min(p.K, kbeg + p.kps);
  const bool vecA = (lda % 4 == 0) && (M % 4 == 0) && ((reinterpret_cast<uintptr_t>(A) & 15) == 0);
  const bool vecB = (ldb % 4 == 0) && (N % 4 == 0) && ((reinterpret_cast<uintptr_t>(B) & 15) == 0);
  const int qa = (M + 3) / 4, qb = (N + 3) / 4;
  float acc[TMB][TNB];
#pragma unroll
  for (int i = 0; i < TMB; i++)
#pragma unroll
    for (int j = 0; j < TNB; j++) acc[i][j] = 0.f;

  float4 ra[MAXQ];
  const int tot_a = R * qa, tot_b = R * qb, tot = tot_a + tot_b;
  // Flat path: dense operands with ld == width (the weight-gradient case): an R-row block of each is
  // one contiguous range, copied float4 by float4 (rows past kend zero-filled by offset compare).
  const bool flat = vecA && vecB && lda == M && ldb == N;
  auto gload = [&](int k0) {
    if (flat) {
      const int rows_ok = max(0, min(R, kend - k0));
      const int lim_a = rows_ok * M / 4, lim_b = rows_ok * N / 4;
      const float4* ga = reinterpret_cast<const float4*>(A + (long long)k0 * lda);
      const float4* gb = reinterpret_cast<const float4*>(B + (long long)k0 * ldb);
#pragma unroll
      for (int j = 0; j < MAXQ; j++) {
        const int idx = tid + j * NTH;
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
        if (idx < tot_a) { if (idx < lim_a) v = __ldg(ga + idx); }
        else if (idx < tot) { if (idx - tot_a < lim_b) v = __ldg(gb + (idx - tot_a)); }
        ra[j] = v;
      }
      return;
    }
#pragma unroll
    for (int j = 0; j < MAXQ; j++) {
      const int idx = tid + j * NTH;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (idx < tot) {
        const bool isA = idx < tot_a;
        const int li = isA ? idx : idx - tot_a;
        const int q = isA ? qa : qb;
        const int r = li / q, c = (li % q) * 4;
        const int k = k0 + r;
        if (k < kend) {
          const float* base = isA ? A + (long long)k * lda : B + (long long)k * ldb;
          const int lim = isA ? M : N;
          if ((isA ? vecA : vecB)) v = __ldg(reinterpret_cast<const float4*>(base + c));
          else {
            v.x = c < lim ? __ldg(base + c) : 0.f;
            v.y = c + 1 < lim ? __ldg(base + c + 1) : 0.f;
            v.z = c + 2 < lim ? __ldg(base + c + 2) : 0.f;
            v.w = c + 3 < lim ? __ldg(base + c + 3) : 0.f;
          }
        }
      }
      ra[j] = v;
    }
  };
  const int sA = flat ? M : Mp, sB = flat ? N : Np;   // staged row strides
  auto sstore = [&](int buf) {
#pragma unroll
    for (int j = 0; j < MAXQ; j++) {
      const int idx = tid + j * NTH;
      if (idx < tot) {
        const bool isA = idx < tot_a;
        const int li = isA ? idx : idx - tot_a;
        if (flat) {
          if (isA) reinterpret_cast<float4*>(As0 + (size_t)buf * R * Mp)[li] = ra[j];
          else reinterpret_cast<float4*>(Bs0 + (size_t)buf * R * Np)[li] = ra[j];
        } else {
          const int q = isA ? qa : qb;
          const int r = li / q, c = (li % q) * 4;
          float* dst = isA ? As0 + ((size_t)buf * R + r) * Mp + c : Bs0 + ((size_t)buf * R + r) * Np + c;
          *reinterpret_cast<float4*>(dst) = ra[j];
        }
      }
    }
  };
  int buf = 0;
  if (kbeg < kend) { gload(kbeg); sstore(0); }
  __syncthreads();
  for (int k0 = kbeg; k0 < kend; k0 += R) {
    const bool more = k0 + R < kend;
    if (more) gload(k0 + R);
    if (active) {
      const float* ab = As0 + (size_t)buf * R * Mp + bm;
      const float* bb = Bs0 + (size_t)buf * R * Np + bn;
      for (int r = grp; r < R; r += G) {
        float av[TMB], bv[TNB];
#pragma unroll
        for (int i = 0; i < TMB; i += 4) {
          const float4 a = *reinterpret_cast<const float4*>(ab + (size_t)r * sA + i);
          av[i] = a.x; av[i + 1] = a.y; av[i + 2] = a.z; av[i + 3] = a.w;
        }
#pragma unroll
        for (int j = 0; j < TNB; j += 4) {
          const float4 b = *reinterpret_cast<const float4*>(bb + (size_t)r * sB + j);
          bv[j] = b.x; bv[j + 1] = b.y; bv[j + 2] = b.z; bv[j + 3] = b.w;
        }
#pragma unroll
        for (int i = 0; i < TMB; i++)
#pragma unroll
          for (int j = 0; j < TNB; j++) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
      }
    }
    if (more) {
      __syncthreads();
      sstore(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }
  // combine row groups in fixed order
  constexpr int BLK = TMB * TNB;
  if (active) {
#pragma unroll
    for (int i = 0; i < TMB; i++)
#pragma unroll
      for (int j = 0; j < TNB; j++) red[(grp * nblk + blk) * BLK + i * TNB + j] = acc[i][j];
  }
  __syncthreads();
  float* out = p.split == 1 ? nullptr : p.ws + (long long)blockIdx.z * M * N;
  for (int e = tid; e < nblk * BLK; e += NTH) {
    const int b = e / BLK, ij = e % BLK, i = ij / TNB, j = ij % TNB;
    const int m = (b / nb) * TMB + i, n = (b % nb) * TNB + j;
    float v = 0.f;
    for (int g = 0; g < G; g++) v += red[(g * nblk + b) * BLK + ij];
    if (m < M && n < N) {
      if (p.split == 1) p.C[(long long)m * p.ldc + n] = v + (p.bias ? __ldg(p.bias + n) : 0.f);
      else out[(long long)m * N + n] = v;
    }
  }
  if (p.split > 1) split_finish(p, 0, 0, 0, M, N);
  orion_signal(sig);
}
}  // namespace atb

// ---------------------------------------------------------------- tall-skinny rows GEMM
// C[M][N] = A[M][K] B for M >> N (N <= 32): 1x1-conv forward into few channels and the data
// gradient of expand convs. HBM-bound on A and C, so each CTA streams a contiguous block of 256 rows
// of A (coalesced 128-bit loads, transposed into shared memory so each thread reads its own row
// conflict-free), B lives in shared memory for the whole CTA (broadcast reads), and each thread
// accumulates its row's N outputs in registers in k order (deterministic, no split).
namespace rows {
constexpr int NTH = 256, KC = 32, NCH = 32, MAXKN = 16384;

// Threads are (row, chunk): each thread owns NCH = 32 consecutive outputs of one row; a CTA holds
// RPC = 256 / nchunk rows (nchunk = ceil(N / 32) <= 4).
template <bool BT>
__global__ void __launch_bounds__(NTH) gemm_rows_kernel(const float* __restrict__ A, long long lda, const float* __restrict__ B,
                                                       long long ldb, float* __restrict__ C, long long ldc,
                                                       const float* __restrict__ bias, int M, int N, int K, OrionSig sig) {
  extern __shared__ __align__(16) float rows_smem[];
  const int NP = (N + 3) & ~3;                    // B rows padded to whole float4
  const int nchunk = (N + NCH - 1) / NCH;
  const int RPC = NTH / nchunk;
  float* Bs = rows_smem;                          // [K][NP]
  float* As = Bs + K * NP;                        // [KC][RPC + 1]
  const int tid = threadIdx.x;
  const int row = tid % RPC, chunk = tid / RPC;
  const bool thr_on = chunk < nchunk;
  const int n0 = chunk * NCH;
  const int nq = thr_on ? (min(NCH, NP - n0) + 3) / 4 : 0;   // float4 columns of this thread
  for (int i = tid; i < K * NP; i += NTH) {
    const int k = i / NP, n = i % NP;
    Bs[i] = n < N ? (BT ? __ldg(B + (long long)n * ldb + k) : __ldg(B + (long long)k * ldb + n)) : 0.f;
  }
  const long long r0 = (long long)blockIdx.x * RPC;
  const int rows_here = (int)min((long long)RPC, (long long)M - r0);
  float4 acc[NCH / 4];
#pragma unroll
  for (int j = 0; j < NCH / 4; j++) acc[j] = make_float4(0.f, 0.f, 0.f, 0.f);
  const bool vec = (lda % 4 == 0) && ((reinterpret_cast<uintptr_t>(A) & 15) == 0);
  for (int k0 = 0; k0 < K; k0 += KC) {
    const int kc = min(KC, K - k0);
    __syncthreads();   // previous chunk consumed (and Bs staged on the first pass)
    if (vec && (kc % 4) == 0) {
      const int q = kc / 4;
      for (int i = tid; i < rows_here * q; i += NTH) {
        const int r = i / q, c = (i % q) * 4;
        const float4 v = __ldg(reinterpret_cast<const float4*>(A + (r0 + r) * lda + k0 + c));
        As[(c + 0) * (RPC + 1) + r] = v.x; As[(c + 1) * (RPC + 1) + r] = v.y;
        As[(c + 2) * (RPC + 1) + r] = v.z; As[(c + 3) * (RPC + 1) + r] = v.w;
      }
    } else {
      for (int i = tid; i < rows_here * kc; i += NTH) {
        const int r = i / kc, c = i % kc;
        As[c * (RPC + 1) + r] = __ldg(A + (r0 + r) * lda + k0 + c);
      }
    }
    __syncthreads();
    if (thr_on && row < rows_here) {
      for (int kk = 0; kk < kc; kk++) {
        const float a = As[kk * (RPC + 1) + row];
        const float4* b = reinterpret_cast<const float4*>(Bs + (k0 + kk) * NP + n0);
#pragma unroll
        for (int j = 0; j < NCH / 4; j++) {
          if (j < nq) {
            const float4 bv = b[j];
            acc[j].x = fmaf(a, bv.x, acc[j].x); acc[j].y = fmaf(a, bv.y, acc[j].y);
            acc[j].z = fmaf(a, bv.z, acc[j].z); acc[j].w = fmaf(a, bv.w, acc[j].w);
          }
        }
      }
    }
  }
  if (thr_on && row < rows_here) {
    float* c = C + (r0 + row) * ldc + n0;
    const bool vc = (N % 4 == 0) && (ldc % 4 == 0) && ((reinterpret_cast<uintptr_t>(C) & 15) == 0) && bias == nullptr;
#pragma unroll
    for (int j = 0; j < NCH / 4; j++) {
      if (j < nq) {
        if (vc) {
          reinterpret_cast<float4*>(c)[j] = acc[j];
        } else {
          const float v[4] = {acc[j].x, acc[j].y, acc[j].z, acc[j].w};
#pragma unroll
          for (int e = 0; e < 4; e++) {
            const int n = n0 + 4 * j + e;
            if (n < N) c[4 * j + e] = v[e] + (bias ? __ldg(bias + n) : 0.f);
          }
        }
      }
    }
  }
  orion_signal(sig);
}
inline int rpc(int N) { return NTH / ((N + NCH - 1) / NCH); }
inline int smem_bytes(int K, int N) { return (K * ((N + 3) & ~3) + KC * (rpc(N) + 1)) * 4; }
}  // namespace rows

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
      // unrolled: four iterations' loads in flight per lane (the loop was one dependent load
      // round trip per 128 columns: 32 us for the ResNet fc at batch 4, ncu)
#pragma unroll 4
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
// cfg: 0/1/2 = FFMA tiles L/M/S; 3/4 = tcgen05 3xTF32 with BN = 128 / 64.

// Skinny A^T B (cfg 5/6/7 = variants V44/V84/V48): the whole M x N fits one CTA's register
// blocks (<= 256 of them), long K.
// First fitting variant in this order. (An 8x8 register-block variant was measured slower than these
// and than the split-K tensor-core path on ResNet-50's 64 x 256 weight gradients, ncu r01.)
int atb_variant(long long M, long long N, long long K) {
  if (K < 4096) return -1;
  if (atb::V44::fits(M, N)) return 5;
  if (atb::V84::fits(M, N)) return 6;
  if (atb::V48::fits(M, N)) return 7;
  return -1;
}
bool atb_ok(long long M, long long N, long long K) { return atb_variant(M, N, K) >= 0; }

Plan plan_atb(long long M, long long N, long long K) {
  Plan pl;
  pl.cfg = atb_variant(M, N, K); pl.bm = (int)M; pl.bn = (int)N; pl.bk = pl.cfg == 5 ? 64 : 32;
  long long split = cdiv(148 * 4, 1);
  long long kmax = K / (4 * pl.bk);
  if (split > kmax) split = kmax;
  if (split < 1) split = 1;
  pl.split = (int)split;
  return pl;
}

Plan plan_gemm(long long M, long long N, long long K) {
  Plan pl;
  const bool tc_ok = M >= 64 && N >= 32 && K >= 64 && M * N * K >= (1LL << 22);
  if (tc_ok) {
    // BN = 128 only when that already yields >= 74 tiles; otherwise BN = 64 doubles the tiles so
    // fewer K splits are needed (each split adds bm*bn*4 bytes the last CTA must re-read).
    const bool wide = N >= 96 && cdiv(M, 128) * cdiv(N, 128) >= 74;
    pl.cfg = wide ? 3 : 4; pl.bm = 128; pl.bn = wide ? 128 : 64; pl.bk = 32;
    long long tiles = cdiv(M, pl.bm) * cdiv(N, pl.bn);
    long long ktiles = cdiv(K, pl.bk);
    long long split = 1;
    if (tiles < 148) {              // one CTA per SM (~196 KB smem each): fill a 148-SM part once,
      split = 148 / tiles;          // never spilling into a second wave
      if (split > ktiles / 4) split = ktiles / 4;   // >= 4 k-tiles per split
      if (split > 128) split = 128;                 // ordered two-level reduction (split_finish) beyond 32
      if (split < 1) split = 1;
    }
    pl.split = (int)split;
    return pl;
  }
  if (M >= 128 && N >= 128 && M * N >= 128LL * 128 * 64) { pl.cfg = 0; pl.bm = 128; pl.bn = 128; pl.bk = 8; }
  else if (M >= 48 && N >= 48) { pl.cfg = 1; pl.bm = 64; pl.bn = 64; pl.bk = 16; }
  else { pl.cfg = 2; pl.bm = 32; pl.bn = 32; pl.bk = 32; }
  long long tiles = cdiv(M, pl.bm) * cdiv(N, pl.bn);
  long long target = 148 * 8;                 // long-K (weight-gradient) GEMMs are HBM-bound: many CTAs
  long long split = 1;
  if (tiles < target) {
    split = cdiv(target, tiles);
    long long kmax = K / (4 * pl.bk);         // >= 4 k-tiles per split
    if (split > kmax) split = kmax;
    if (split > 1008) split = 1008;                 // two-level reduction: <= 32 groups of <= 32
    if (split < 1) split = 1;
  }
  pl.split = (int)split;
  return pl;
}

uint64_t ws_bytes_for(const Plan& pl, long long M, long long N) {
  if (pl.split <= 1) return 0;
  uint64_t parts = (uint64_t)pl.split;
  parts += (uint64_t)split_groups(pl.split);   // group partials
  return WS_TICKET_BYTES + parts * M * N * 4;
}

template <class LA, class LB>
const void* kernel_for(int cfg) {
  switch (cfg) {
    case 0: return (const void*)gemm_kernel<TileL, LA, LB>;
    case 1: return (const void*)gemm_kernel<TileM, LA, LB>;
    case 2: return (const void*)gemm_kernel<TileS, LA, LB>;
    case 3: return (const void*)tc::gemm_tc_kernel<128, LA, LB>;
    default: return (const void*)tc::gemm_tc_kernel<64, LA, LB>;
  }
}

// Opt the tcgen05 kernels into > 48 KB dynamic shared memory once per instantiation.
template <int BN, class LA, class LB>
bool tc_prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  bool ok = cudaFuncSetAttribute((const void*)tc::gemm_tc_kernel<BN, LA, LB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 tc::TcCfg<BN>::SMEM) == cudaSuccess;
  if (ok) done.store(1, std::memory_order_release);
  return ok;
}

// Geometry of a tiled launch; falls back to split 1 when the caller's workspace is too small.
template <class LA, class LB>
void tiled_geom(LaunchGeom* g, long long M, long long N, long long K, uint64_t ws_ptr, uint64_t ws_bytes) {
  Plan pl = plan_gemm(M, N, K);
  if (pl.split > 1 && (ws_ptr == 0 || ws_bytes < ws_bytes_for(pl, M, N))) pl.split = 1;
  g->grid = dim3((unsigned)cdiv(N, pl.bn), (unsigned)cdiv(M, pl.bm), (unsigned)pl.split);
  g->func = kernel_for<LA, LB>(pl.cfg);
  if (pl.cfg == 3) { tc_prepare<128, LA, LB>(); g->block = dim3(tc::NTHR); g->smem = tc::TcCfg<128>::SMEM; g->pipe = ORION_PIPE_TF32X3; }
  else if (pl.cfg == 4) { tc_prepare<64, LA, LB>(); g->block = dim3(tc::NTHR); g->smem = tc::TcCfg<64>::SMEM; g->pipe = ORION_PIPE_TF32X3; }
  else { g->block = dim3(NT); g->smem = 0; }
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
  } else if (g.func == (const void*)gemm_kernel<TileS, LA, LB>) {
    gemm_kernel<TileS, LA, LB><<<g.grid, g.block, 0, s>>>(make_params(M, N, K, C, ldc, bias, split, ws, TileS::BK), la, lb, sig);
  } else if (g.func == (const void*)tc::gemm_tc_kernel<128, LA, LB>) {
    if (!tc_prepare<128, LA, LB>()) return ORION_E_CUDA;
    tc::gemm_tc_kernel<128, LA, LB><<<g.grid, g.block, g.smem, s>>>(make_params(M, N, K, C, ldc, bias, split, ws, tc::BK), la, lb, sig);
  } else {
    if (!tc_prepare<64, LA, LB>()) return ORION_E_CUDA;
    tc::gemm_tc_kernel<64, LA, LB><<<g.grid, g.block, g.smem, s>>>(make_params(M, N, K, C, ldc, bias, split, ws, tc::BK), la, lb, sig);
  }
  return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
}

// ---------------------------------------------------------------- few-input-channel convs (stem)
// The network stem (C = 3 input channels) makes a poor implicit GEMM (K = R*S*C = 27). Forward: one
// thread per output pixel gathers its R*S*C window into registers and produces all K outputs
// (weights in shared memory, 128-bit stores of the output row). (The stem's weight gradient stays
// on the tiled split-K path, which measured faster.)
namespace smallc {
constexpr int NTH = 256, MAXK = 64;

template <int R, int S, int C, int K>
__global__ void __launch_bounds__(NTH) conv_fwd_smallc_kernel(const float* __restrict__ x, const float* __restrict__ w,
                                                              float* __restrict__ y, ConvShape s, OrionSig sig) {
  constexpr int RSC = R * S * C, SC = S * C;
  // weights transposed to [rsc][k]: one warp-uniform 128-bit load feeds four outputs' FMAs, issued
  // as two packed FFMA2 (each output still sums its RSC products in rsc order, as fmaf would). The
  // window is gathered one filter row (S*C values) at a time, so the 7x7x3 ResNet stem fits in
  // registers too. (Measured on the 3x3 stem: as fast as the scalar form -- it is bound by its L1
  // traffic, ncu "Mem Busy" 91 %; a shared-memory-staged variant with coalesced row stores was
  // slower, 171 vs 118 us.)
  extern __shared__ __align__(16) float wt[];   // [RSC][K]
  for (int i = threadIdx.x; i < K * RSC; i += NTH) wt[(i % RSC) * K + i / RSC] = __ldg(w + i);
  __syncthreads();
  const float4* wt4 = reinterpret_cast<const float4*>(wt);
  const long long npix = (long long)s.N * s.P * s.Q;
  for (long long pix = (long long)blockIdx.x * NTH + threadIdx.x; pix < npix; pix += (long long)gridDim.x * NTH) {
    const int q = (int)(pix % s.Q); const long long t = pix / s.Q;
    const int p = (int)(t % s.P); const int n = (int)(t / s.P);
    float2 acc[K / 2];
#pragma unroll
    for (int j = 0; j < K / 2; j++) acc[j] = make_float2(0.f, 0.f);
#pragma unroll 1
    for (int r = 0; r < R; r++) {
      const int h = p * s.stride - s.pad + r;
      float patch[SC];
#pragma unroll
      for (int u = 0; u < S; u++) {
        const int ww = q * s.stride - s.pad + u;
        const bool ok = (unsigned)h < (unsigned)s.H && (unsigned)ww < (unsigned)s.W;
        const float* src = x + (((long long)n * s.H + (ok ? h : 0)) * s.W + (ok ? ww : 0)) * C;
#pragma unroll
        for (int c = 0; c < C; c++) patch[u * C + c] = ok ? __ldg(src + c) : 0.f;
      }
#pragma unroll
      for (int i = 0; i < SC; i++) {
#pragma unroll
        for (int kq = 0; kq < K / 4; kq++) {
          const float4 w4 = wt4[(r * SC + i) * (K / 4) + kq];
          ffma2(acc[2 * kq], patch[i], make_float2(w4.x, w4.y));
          ffma2(acc[2 * kq + 1], patch[i], make_float2(w4.z, w4.w));
        }
      }
    }
    float4* dst = reinterpret_cast<float4*>(y + pix * K);
#pragma unroll
    for (int kq = 0; kq < K / 4; kq++) dst[kq] = make_float4(acc[2 * kq].x, acc[2 * kq].y, acc[2 * kq + 1].x, acc[2 * kq + 1].y);
  }
  orion_signal(sig);
}

// specialised for the 3x3, 3-channel stem (the only few-channel conv of the workloads)
inline bool fwd3_ok(const ConvShape& s) { return s.C == 3 && s.R == 3 && s.S == 3 && s.K == 32; }   // MobileNetV2
inline bool fwd7_ok(const ConvShape& s) { return s.C == 3 && s.R == 7 && s.S == 7 && s.K == 64; }   // ResNet
inline bool fwd_ok(const ConvShape& s) { return fwd3_ok(s) || fwd7_ok(s); }

// Weight gradient of a few-input-channel stem (ResNet 7x7x3 / MobileNetV2 3x3x3):
// dw[k][r][s][c] = sum_{n,p,q} dy[n,p,q,k] x[n, p*st-pad+r, q*st-pad+s, c]. As an implicit GEMM the
// B operand (im2col of x, C = 3) cannot be loaded in 16-byte pieces and the problem has only
// K x RSC = 64 x 147 outputs over 802816-long sums. Here a CTA walks tiles of QT consecutive
// output pixels of one output row: the tile's dy rows (QT x K, contiguous) and the x window it
// touches (R rows x ((QT-1)*st + S) columns x C, contiguous per row) are staged in shared memory
// (the next tile's loads held in registers while the current one is multiplied), and each thread
// owns a 4 (k) x <= WG_MAXR (rsc) register block. Partials (fp64) of the G CTAs (a shape-only
// count) are combined in CTA order (combine_splits), so results are deterministic.
constexpr int WG_QT = 32, WG_KPT = 4, WG_MAXR = 10, WG_G = 296;   // two CTAs per SM of a full B200
// (Measured and reverted: eight resident waves of the 7x7 stem's weight gradient -- each CTA living
// ~0.1 ms instead of the whole 0.9 ms op at ResNet-50's training batch -- cost 891 -> 978 us and left
// config 3's HP p99 where it was, 1.29x vs 1.31x.)
constexpr int WG1_G = WG_G;
constexpr int WG_PF_DY = WG_QT * MAXK / 4 / NTH, WG_PF_X = 8;   // per-thread prefetch registers
__host__ __device__ inline int wg_wwin(const ConvShape& s) { return (WG_QT - 1) * s.stride + s.S; }
__host__ __device__ inline int wg_xwin(const ConvShape& s) { return s.R * wg_wwin(s) * s.C; }
inline long long wg_tiles(const ConvShape& s) { return (long long)s.N * s.P * ((s.Q + WG_QT - 1) / WG_QT); }
inline int wg_ctas(const ConvShape& s) { return (int)(wg_tiles(s) < WG1_G ? wg_tiles(s) : WG1_G); }
// register-block width (rsc per thread) of the launch: 10 for the ResNet stem (147 / 16 groups)
inline int wg_nr(const ConvShape& s) { return (s.R * s.S * s.C + NTH / (s.K / WG_KPT) - 1) / (NTH / (s.K / WG_KPT)); }
// Taken for the large stems (R*S*C >= 64, e.g. ResNet's 7x7x3); the 3x3x3 MobileNetV2 stem has too
// few products per staged value and stays on the tiled split-K path.
inline bool wgrad_ok(const ConvShape& s) {
  const int kg = s.K / WG_KPT, rsc = s.R * s.S * s.C;
  return s.C <= 4 && s.K % WG_KPT == 0 && s.K <= MAXK && (kg & (kg - 1)) == 0 && rsc >= 64 && wg_nr(s) >= 8 && wg_nr(s) <= WG_MAXR &&
         wg_xwin(s) <= NTH * WG_PF_X && s.stride <= 2;
}
inline bool wgrad2_ok(const ConvShape& s);
inline int w2_ctas(const ConvShape& s);
inline uint64_t wgrad_ws_bytes(const ConvShape& s) {
  const uint64_t V = (uint64_t)s.K * s.R * s.S * s.C;
  const int G = wg_ctas(s), G2 = w2_ctas(s);
  // 7x7 kernel: fp32 partials + fp64 group rows; 3x3 kernel: fp64 partials + group rows
  const uint64_t b1 = WS_TICKET_BYTES + ((uint64_t)G * V * 4 + 15) / 16 * 16 + (uint64_t)(combine_rows(G) + 1) * V * 8;
  const uint64_t b2 = WS_TICKET_BYTES + (uint64_t)(G2 + combine_rows(G2) + 1) * V * 8;
  return b1 > b2 ? b1 : b2;
}

template <int NR>
__global__ void __launch_bounds__(NTH, 2) conv_wgrad_smallc_kernel(const float* __restrict__ x, const float* __restrict__ dy,
                                                                   float* __restrict__ dw, ConvShape s, unsigned char* ws, OrionSig sig) {
  extern __shared__ __align__(16) float wsm[];
  const int K = s.K, RSC = s.R * s.S * s.C, WW = wg_wwin(s), XW = wg_xwin(s);
  float* dys = wsm;                      // [WG_QT][K]
  float* xs = wsm + WG_QT * K;           // [R][WW][C]
  const int kgroups = K / WG_KPT, rgroups = NTH / kgroups;
  const int kg = threadIdx.x % kgroups, rg = threadIdx.x / kgroups;
  int off[NR];
#pragma unroll
  for (int i = 0; i < NR; i++) {
    const int j = rg + rgroups * i;
    if (j < RSC) {
      const int c = j % s.C, t = j / s.C, u = t % s.S, r = t / s.S;
      off[i] = (r * WW + u) * s.C + c;
    } else {
      off[i] = 0;   // padding slot: accumulates garbage that is never stored (no branch in the hot loop)
    }
  }
  float2 acc2[WG_KPT / 2][NR];   // (k, k+1) pairs: packed FFMA2, each lane rounded as fmaf
#pragma unroll
  for (int a = 0; a < WG_KPT / 2; a++)
#pragma unroll
    for (int i = 0; i < NR; i++) acc2[a][i] = make_float2(0.f, 0.f);
  const int qtiles = (s.Q + WG_QT - 1) / WG_QT;
  const long long T = (long long)s.N * s.P * qtiles;
  float4 pdy[WG_PF_DY];
  float px[WG_PF_X];
#define WG_FETCH(TT)                                                                                                    \
  {                                                                                                                     \
    const long long t_ = (TT);                                                                                          \
    const int qt = (int)(t_ % qtiles); const long long np = t_ / qtiles;                                                \
    const int p = (int)(np % s.P), n = (int)(np / s.P);                                                                 \
    const int q0 = qt * WG_QT, qn = min(WG_QT, s.Q - q0);                                                               \
    const float4* src = reinterpret_cast<const float4*>(dy + (((long long)n * s.P + p) * s.Q + q0) * K);                \
    _Pragma("unroll") for (int e = 0; e < WG_PF_DY; e++) {                                                              \
      const int idx = threadIdx.x + e * NTH;                                                                            \
      pdy[e] = (idx * 4 < qn * K) ? __ldg(src + idx) : make_float4(0.f, 0.f, 0.f, 0.f);                                  \
    }                                                                                                                   \
    const int h0 = p * s.stride - s.pad, w0 = q0 * s.stride - s.pad;                                                    \
    _Pragma("unroll") for (int e = 0; e < WG_PF_X; e++) {                                                               \
      const int idx = threadIdx.x + e * NTH;                                                                            \
      float v = 0.f;                                                                                                    \
      if (idx < XW) {                                                                                                   \
        const int c = idx % s.C, t2 = idx / s.C, u = t2 % WW, r = t2 / WW;                                              \
        const int h = h0 + r, w = w0 + u;                                                                               \
        if ((unsigned)h < (unsigned)s.H && (unsigned)w < (unsigned)s.W) v = __ldg(x + (((long long)n * s.H + h) * s.W + w) * s.C + c); \
      }                                                                                                                 \
      px[e] = v;                                                                                                        \
    }                                                                                                                   \
  }
  long long t = blockIdx.x;
  if (t < T) WG_FETCH(t);
  for (; t < T; t += gridDim.x) {
    __syncthreads();                                    // previous tile's compute done
#pragma unroll
    for (int e = 0; e < WG_PF_DY; e++) {
      const int idx = threadIdx.x + e * NTH;
      if (idx * 4 < WG_QT * K) reinterpret_cast<float4*>(dys)[idx] = pdy[e];
    }
#pragma unroll
    for (int e = 0; e < WG_PF_X; e++) {
      const int idx = threadIdx.x + e * NTH;
      if (idx < XW) xs[idx] = px[e];
    }
    __syncthreads();
    if (t + gridDim.x < T) WG_FETCH(t + gridDim.x);    // next tile's loads in flight during the math
    const int xstep = s.stride * s.C;
#pragma unroll 4
    for (int i = 0; i < WG_QT; i++) {                   // zero dy rows beyond Q contribute nothing
      const float4 d = *reinterpret_cast<const float4*>(dys + i * K + kg * WG_KPT);
      const float* xr = xs + i * xstep;
#pragma unroll
      for (int j = 0; j < NR; j++) {
        const float xv = xr[off[j]];
        ffma2(acc2[0][j], xv, make_float2(d.x, d.y));
        ffma2(acc2[1][j], xv, make_float2(d.z, d.w));
      }
    }
  }
  // partial of this CTA -> workspace (fp64), ordered combine over the G CTAs
  const long long V = (long long)K * RSC;
  unsigned int* tk = reinterpret_cast<unsigned int*>(ws);
  float* part = reinterpret_cast<float*>(ws + WS_TICKET_BYTES);
  const int G = gridDim.x;
  double* gpart = reinterpret_cast<double*>(ws + WS_TICKET_BYTES + ((uint64_t)G * V * 4 + 15) / 16 * 16);
  double* out = gpart + (long long)combine_rows(G) * V;
#pragma unroll
  for (int j = 0; j < NR; j++) {
    const int jj = rg + rgroups * j;
    if (jj < RSC) {
#pragma unroll
      for (int a = 0; a < WG_KPT; a++)
        part[(long long)blockIdx.x * V + (long long)(kg * WG_KPT + a) * RSC + jj] = (a & 1) ? acc2[a / 2][j].y : acc2[a / 2][j].x;
    }
  }
  __shared__ double scratch[NTH];
  if (combine_splits(tk, part, gpart, V, G, blockIdx.x, (int)V, out, scratch)) {
    for (long long v = threadIdx.x; v < V; v += NTH) dw[v] = (float)__ldcg(out + v);
  }
  orion_signal(sig);
}
#undef WG_FETCH

// Variant for the 3x3x3 / 32-filter stem (MobileNetV2): the 864 outputs are few and each value is
// used by few products, so a whole warp covers all outputs of one pixel — lane = (k-quad kg < 8,
// rsc subset rs < 4), 4 x 7 register block — and the 8 warps of a CTA take interleaved pixels of the
// staged 32-pixel tile; warp partials are summed in warp order, CTA partials (fp64) in CTA order.
constexpr int W2_NR = 7, W2_QT = 112, W2_PF_X = 8;   // a whole MobileNetV2 stem output row per tile
__host__ __device__ inline int w2_wwin(const ConvShape& s) { return (W2_QT - 1) * s.stride + s.S; }
__host__ __device__ inline int w2_xwin(const ConvShape& s) { return s.R * w2_wwin(s) * s.C; }
inline bool wgrad2_ok(const ConvShape& s) {
  return s.C <= 4 && s.K == 32 && s.R * s.S * s.C <= 4 * W2_NR && w2_xwin(s) <= NTH * W2_PF_X && s.stride <= 2;
}
__global__ void __launch_bounds__(NTH, 2) conv_wgrad_smallc2_kernel(const float* __restrict__ x, const float* __restrict__ dy,
                                                                    float* __restrict__ dw, ConvShape s, unsigned char* ws, OrionSig sig) {
  extern __shared__ __align__(16) float wsm[];
  constexpr int K = 32;
  const int RSC = s.R * s.S * s.C, WW = w2_wwin(s), XW = w2_xwin(s);
  float* dys = wsm;                      // [W2_QT][K]
  float* xs = wsm + W2_QT * K;           // [R][WW][C]
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const int kg = lane % 8, rs = lane / 8;
  int off[W2_NR];
#pragma unroll
  for (int i = 0; i < W2_NR; i++) {
    const int j = rs + 4 * i;
    if (j < RSC) {
      const int c = j % s.C, t = j / s.C, u = t % s.S, r = t / s.S;
      off[i] = (r * WW + u) * s.C + c;
    } else {
      off[i] = 0;   // padding slot, never stored
    }
  }
  float2 acc2[2][W2_NR];   // acc2[a2][j] = outputs (k = kg*4 + 2*a2, +1) of rsc slot j
#pragma unroll
  for (int a = 0; a < 2; a++)
#pragma unroll
    for (int i = 0; i < W2_NR; i++) acc2[a][i] = make_float2(0.f, 0.f);
  const int qtiles = (s.Q + W2_QT - 1) / W2_QT;
  const long long T = (long long)s.N * s.P * qtiles;
  constexpr int PF_DY = (W2_QT * K / 4 + NTH - 1) / NTH;   // 4 float4 per thread
  float4 pdy[PF_DY];
  float px[W2_PF_X];
#define W2_FETCH(TT)                                                                                                    \
  {                                                                                                                     \
    const long long t_ = (TT);                                                                                          \
    const int qt = (int)(t_ % qtiles); const long long np = t_ / qtiles;                                                \
    const int p = (int)(np % s.P), n = (int)(np / s.P);                                                                 \
    const int q0 = qt * W2_QT, qn = min(W2_QT, s.Q - q0);                                                               \
    const float4* src = reinterpret_cast<const float4*>(dy + (((long long)n * s.P + p) * s.Q + q0) * K);                \
    _Pragma("unroll") for (int e = 0; e < PF_DY; e++) {                                                                 \
      const int idx = threadIdx.x + e * NTH;                                                                            \
      pdy[e] = (idx * 4 < qn * K) ? __ldg(src + idx) : make_float4(0.f, 0.f, 0.f, 0.f);                                  \
    }                                                                                                                   \
    const int h0 = p * s.stride - s.pad, w0 = q0 * s.stride - s.pad;                                                    \
    _Pragma("unroll") for (int e = 0; e < W2_PF_X; e++) {                                                               \
      const int idx = threadIdx.x + e * NTH;                                                                            \
      float v = 0.f;                                                                                                    \
      if (idx < XW) {                                                                                                   \
        const int c = idx % s.C, t2 = idx / s.C, u = t2 % WW, r = t2 / WW;                                              \
        const int h = h0 + r, w = w0 + u;                                                                               \
        if ((unsigned)h < (unsigned)s.H && (unsigned)w < (unsigned)s.W) v = __ldg(x + (((long long)n * s.H + h) * s.W + w) * s.C + c); \
      }                                                                                                                 \
      px[e] = v;                                                                                                        \
    }                                                                                                                   \
  }
  long long t = blockIdx.x;
  if (t < T) W2_FETCH(t);
  for (; t < T; t += gridDim.x) {
    __syncthreads();
#pragma unroll
    for (int e = 0; e < PF_DY; e++)
      if (threadIdx.x + e * NTH < W2_QT * K / 4) reinterpret_cast<float4*>(dys)[threadIdx.x + e * NTH] = pdy[e];
#pragma unroll
    for (int e = 0; e < W2_PF_X; e++) {
      const int idx = threadIdx.x + e * NTH;
      if (idx < XW) xs[idx] = px[e];
    }
    __syncthreads();
    if (t + gridDim.x < T) W2_FETCH(t + gridDim.x);
    const int xstep = s.stride * s.C;
#pragma unroll 2
    for (int i = warp; i < W2_QT; i += NTH / 32) {
      const float4 d = *reinterpret_cast<const float4*>(dys + i * K + kg * 4);
      const float* xr = xs + i * xstep;
#pragma unroll
      for (int j = 0; j < W2_NR; j++) {
        const float xv = xr[off[j]];
        ffma2(acc2[0][j], xv, make_float2(d.x, d.y));   // (k, k+1) pairs: packed FFMA2, same rounding as fmaf
        ffma2(acc2[1][j], xv, make_float2(d.z, d.w));
      }
    }
  }
  __syncthreads();
  // warp partials -> shared [8][K * RSC] (reusing the staging area), summed in warp order
  const int V = K * RSC;
  float* wp = wsm;
#pragma unroll
  for (int j = 0; j < W2_NR; j++) {
    const int jj = rs + 4 * j;
    if (jj < RSC) {
#pragma unroll
      for (int a = 0; a < 4; a++) wp[warp * V + (kg * 4 + a) * RSC + jj] = (a & 1) ? acc2[a / 2][j].y : acc2[a / 2][j].x;
    }
  }
  __syncthreads();
  unsigned int* tk = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  const int G = gridDim.x;
  for (int v = threadIdx.x; v < V; v += NTH) {
    double sum = 0.0;
    for (int w = 0; w < NTH / 32; w++) sum += (double)wp[w * V + v];
    part[(long long)blockIdx.x * V + v] = sum;
  }
  double* gpart = part + (long long)G * V;
  double* out = gpart + (long long)combine_rows(G) * V;
  __shared__ double scratch[NTH];
  if (combine_splits(tk, part, gpart, V, G, blockIdx.x, V, out, scratch)) {
    for (int v = threadIdx.x; v < V; v += NTH) dw[v] = (float)__ldcg(out + v);
  }
  orion_signal(sig);
}
#undef W2_FETCH
inline int w2_ctas(const ConvShape& s) {
  const long long t = (long long)s.N * s.P * ((s.Q + W2_QT - 1) / W2_QT);
  return (int)(t < WG_G ? t : WG_G);
}
inline int wgrad2_smem(const ConvShape& s) {
  const int stage = W2_QT * 32 + w2_xwin(s), red = (NTH / 32) * 32 * s.R * s.S * s.C;
  return (stage > red ? stage : red) * 4;
}

inline const void* wgrad_fn(const ConvShape& s) {
  switch (wg_nr(s)) {
    case 8: return (const void*)conv_wgrad_smallc_kernel<8>;
    case 9: return (const void*)conv_wgrad_smallc_kernel<9>;
    default: return (const void*)conv_wgrad_smallc_kernel<10>;
  }
}
}  // namespace smallc

}  // namespace

// Workspace bytes a tiled GEMM of this (M, N, K) needs for its K split (0 if no split). Conv ops
// pass their implicit-GEMM dims: fwd (N*P*Q, K, R*S*C), dgrad (N*H*W, C, R*S*K), wgrad (K, R*S*C, N*P*Q).
extern "C" uint64_t orion_gemm_workspace_bytes(uint64_t M, uint64_t N, uint64_t K) {
  Plan pl = plan_gemm((long long)M, (long long)N, (long long)K);
  uint64_t b = ws_bytes_for(pl, (long long)M, (long long)N);
  if (atb_ok((long long)M, (long long)N, (long long)K)) {   // A^T B callers may take the skinny kernel
    uint64_t b2 = ws_bytes_for(plan_atb((long long)M, (long long)N, (long long)K), (long long)M, (long long)N);
    if (b2 > b) b = b2;
  }
  const uint64_t b3 = wgs_ws_bytes((long long)M, (long long)N, (long long)K);   // ... or the streaming one
  if (b3 > b) b = b3;
  const uint64_t b4 = atc_ws_bytes((long long)M, (long long)N, (long long)K);   // ... or the tensor-core one
  if (b4 > b) b = b4;
  const uint64_t b5 = ats_ws_bytes((long long)M, (long long)N, (long long)K);   // ... or the streaming tensor-core one
  if (b5 > b) b = b5;
  return b;
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
  if ((flags == 0 || flags == 2) &&
      tmk::ok(M, N, K, (long long)a[7], (long long)a[8], (long long)a[9], (const float*)a[0], (const float*)a[1], (const float*)a[2])) {
    tmk::geom(g, M, N, flags == 0);   // streaming shapes, TMA-fed
    return 0;
  }
  if ((flags == 0 || flags == 2) && tcm::ok(M, N, K)) {   // streaming shapes: multi-tile tcgen05 kernel
    if (flags == 2) tcm::geom<ADense, BDenseT>(g, M, N);
    else tcm::geom<ADense, BDense>(g, M, N);
    return 0;
  }
  if ((flags == 0 || flags == 2) && M >= 4096 && N <= 32 && K * ((N + 3) & ~3) <= rows::MAXKN) {
    const void* f = flags == 2 ? (const void*)rows::gemm_rows_kernel<true> : (const void*)rows::gemm_rows_kernel<false>;
    static std::atomic<int> attr{0};
    if (!attr.load()) {
      if (cudaFuncSetAttribute((const void*)rows::gemm_rows_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (rows::MAXKN + rows::KC * (rows::NTH + 1)) * 4) != cudaSuccess ||
          cudaFuncSetAttribute((const void*)rows::gemm_rows_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (rows::MAXKN + rows::KC * (rows::NTH + 1)) * 4) != cudaSuccess)
        return ORION_E_CUDA;
      attr.store(1);
    }
    g->grid = dim3((unsigned)cdiv(M, rows::rpc((int)N))); g->block = dim3(rows::NTH); g->smem = rows::smem_bytes((int)K, (int)N); g->func = f;
    return 0;
  }
  if ((flags == 2 || flags == 0) && cvf_gemm_try_geom(a, g)) return 0;   // dense GEMM, TMA-fed tcgen05 (cvf.cu)
  if (flags == 1 && ats_try_geom(a, g)) return 0;   // long-K narrow A^T B streamed into tcgen05 (ats.cu)
  if (flags == 1 && atc_try_geom(a, g)) return 0;   // compute-dense A^T B on tcgen05 (atc.cu)
  if (flags == 1 && wgs_try_geom(a, g)) return 0;   // TMA-fed streaming A^T B (wgs.cu)
  if (flags == 1 && atb_ok(M, N, K)) {
    Plan pl = plan_atb(M, N, K);
    if (pl.split > 1 && (a[11] == 0 || a[12] < ws_bytes_for(pl, M, N))) pl.split = 1;
    static std::atomic<int> attr{0};
    if (!attr.load()) {
      if (cudaFuncSetAttribute((const void*)atb::gemm_atb_kernel<atb::V44, 4, 4, 64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               atb::V44::smem_bytes(128, 128)) != cudaSuccess ||
          cudaFuncSetAttribute((const void*)atb::gemm_atb_kernel<atb::V84, 8, 4, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               atb::V84::smem_bytes(192, 64)) != cudaSuccess ||
          cudaFuncSetAttribute((const void*)atb::gemm_atb_kernel<atb::V48, 4, 8, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               atb::V48::smem_bytes(64, 192)) != cudaSuccess)
        return ORION_E_CUDA;
      attr.store(1);
    }
    g->grid = dim3(1, 1, (unsigned)pl.split); g->block = dim3(atb::NTH);
    if (pl.cfg == 5) { g->smem = atb::V44::smem_bytes((int)M, (int)N); g->func = (const void*)atb::gemm_atb_kernel<atb::V44, 4, 4, 64>; }
    else if (pl.cfg == 6) { g->smem = atb::V84::smem_bytes((int)M, (int)N); g->func = (const void*)atb::gemm_atb_kernel<atb::V84, 8, 4, 32>; }
    else { g->smem = atb::V48::smem_bytes((int)M, (int)N); g->func = (const void*)atb::gemm_atb_kernel<atb::V48, 4, 8, 32>; }
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
  if (atc_is(g.func)) return atc_launch(a, g, sig, s);
  if (ats_is(g.func)) return ats_launch(a, g, sig, s);
  if (cvf_is(g.func)) return cvf_gemm_launch(a, g, sig, s);
  if (wgs_is(g.func)) return wgs_launch(a, g, sig, s);
  if (tmk::is(g.func)) return tmk::launch(g, M, N, K, C, ldc, bias, A, lda, B, ldb, flags == 0, sig, s);
  if (tcm::is<ADense, BDenseT>(g.func))
    return tcm::launch(g, M, N, K, C, ldc, bias, ADense{A, lda}, BDenseT{B, ldb}, sig, s);
  if (tcm::is<ADense, BDense>(g.func))
    return tcm::launch(g, M, N, K, C, ldc, bias, ADense{A, lda}, BDense{B, ldb}, sig, s);
  if (g.func == (const void*)rows::gemm_rows_kernel<true> || g.func == (const void*)rows::gemm_rows_kernel<false>) {
    if (flags == 2)
      rows::gemm_rows_kernel<true><<<g.grid, g.block, g.smem, s>>>(A, lda, B, ldb, C, ldc, bias, (int)M, (int)N, (int)K, sig);
    else
      rows::gemm_rows_kernel<false><<<g.grid, g.block, g.smem, s>>>(A, lda, B, ldb, C, ldc, bias, (int)M, (int)N, (int)K, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  if (g.func == (const void*)atb::gemm_atb_kernel<atb::V44, 4, 4, 64>) {
    atb::gemm_atb_kernel<atb::V44, 4, 4, 64><<<g.grid, g.block, g.smem, s>>>(make_params(M, N, K, C, ldc, bias, (int)g.grid.z, ws, 64), A, lda, B, ldb, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  if (g.func == (const void*)atb::gemm_atb_kernel<atb::V84, 8, 4, 32>) {
    atb::gemm_atb_kernel<atb::V84, 8, 4, 32><<<g.grid, g.block, g.smem, s>>>(make_params(M, N, K, C, ldc, bias, (int)g.grid.z, ws, 32), A, lda, B, ldb, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  if (g.func == (const void*)atb::gemm_atb_kernel<atb::V48, 4, 8, 32>) {
    atb::gemm_atb_kernel<atb::V48, 4, 8, 32><<<g.grid, g.block, g.smem, s>>>(make_params(M, N, K, C, ldc, bias, (int)g.grid.z, ws, 32), A, lda, B, ldb, sig);
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
  if (smallc::fwd_ok(s)) {
    static std::atomic<int> attr{0};
    if (!attr.load()) {
      if (cudaFuncSetAttribute((const void*)smallc::conv_fwd_smallc_kernel<7, 7, 3, 64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               7 * 7 * 3 * 64 * 4) != cudaSuccess) {
        (void)cudaGetLastError();
        return ORION_E_CUDA;
      }
      attr.store(1);
    }
    long long ctas = cdiv((long long)s.N * s.P * s.Q, smallc::NTH);
    g->grid = dim3((unsigned)(ctas < 148 * 16 ? ctas : 148 * 16)); g->block = dim3(smallc::NTH);
    g->smem = s.R * s.S * s.C * s.K * 4;
    g->func = smallc::fwd3_ok(s) ? (const void*)smallc::conv_fwd_smallc_kernel<3, 3, 3, 32> : (const void*)smallc::conv_fwd_smallc_kernel<7, 7, 3, 64>;
    return 0;
  }
  if (cvf_conv_try_geom(a, g)) return 0;   // TMA im2col boxes straight into tcgen05 (cvf.cu)
  tiled_geom<AIm2col, BDenseT>(g, (long long)s.N * s.P * s.Q, s.K, (long long)s.R * s.S * s.C, a[14], a[15]);
  return 0;
}
int conv_fwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  if (cvf_is(g.func)) return cvf_conv_launch(a, g, sig, st);
  ConvShape s = conv_shape(a);
  if (g.func == (const void*)smallc::conv_fwd_smallc_kernel<3, 3, 3, 32>) {
    smallc::conv_fwd_smallc_kernel<3, 3, 3, 32><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  if (g.func == (const void*)smallc::conv_fwd_smallc_kernel<7, 7, 3, 64>) {
    smallc::conv_fwd_smallc_kernel<7, 7, 3, 64><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s, sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
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

extern "C" uint64_t orion_conv_wgrad_workspace_bytes(uint64_t N, uint64_t H, uint64_t W, uint64_t C, uint64_t K, uint64_t R,
                                                     uint64_t S, uint64_t stride, uint64_t pad) {
  ConvShape s{(int)N, (int)H, (int)W, (int)C, (int)K, (int)R, (int)S, (int)stride, (int)pad,
              (int)((H + 2 * pad - R) / stride + 1), (int)((W + 2 * pad - S) / stride + 1)};
  uint64_t b = orion_gemm_workspace_bytes(K, R * S * C, (uint64_t)N * s.P * s.Q);
  if (smallc::wgrad_ok(s) || smallc::wgrad2_ok(s)) {
    const uint64_t b2 = smallc::wgrad_ws_bytes(s);
    if (b2 > b) b = b2;
  }
  const uint64_t b3 = atc_conv_ws_bytes(N, H, W, C, K, R, S, stride, pad);   // tcgen05 path (atc.cu)
  if (b3 > b) b = b3;
  return b;
}

int conv_wgrad_geom(const uint64_t* a, LaunchGeom* g) {
  ConvShape s = conv_shape(a);
  if (smallc::wgrad2_ok(s) && a[14] != 0 && a[15] >= smallc::wgrad_ws_bytes(s)) {
    static std::atomic<int> attr{0};
    if (!attr.load()) {
      if (cudaFuncSetAttribute((const void*)smallc::conv_wgrad_smallc2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024) !=
          cudaSuccess)
        return ORION_E_CUDA;
      attr.store(1);
    }
    g->grid = dim3((unsigned)smallc::w2_ctas(s)); g->block = dim3(smallc::NTH);
    g->smem = smallc::wgrad2_smem(s);
    g->func = (const void*)smallc::conv_wgrad_smallc2_kernel;
    return 0;
  }
  if (smallc::wgrad_ok(s) && a[14] != 0 && a[15] >= smallc::wgrad_ws_bytes(s)) {
    g->grid = dim3((unsigned)smallc::wg_ctas(s)); g->block = dim3(smallc::NTH);
    g->smem = (smallc::WG_QT * s.K + smallc::wg_xwin(s)) * 4;   // <= 24 KB
    g->func = smallc::wgrad_fn(s);
    return 0;
  }
  if (atc_conv_try_geom(a, g)) return 0;   // TMA 4-D boxes straight into tcgen05 (atc.cu)
  tiled_geom<ADenseT, BWgrad>(g, s.K, (long long)s.R * s.S * s.C, (long long)s.N * s.P * s.Q, a[14], a[15]);
  return 0;
}
int conv_wgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  if (atc_conv_is(g.func)) return atc_conv_launch(a, g, sig, st);
  ConvShape s = conv_shape(a);
  if (g.func == (const void*)smallc::conv_wgrad_smallc2_kernel) {
    smallc::conv_wgrad_smallc2_kernel<<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s,
                                                                       (unsigned char*)a[14], sig);
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  if (smallc::wgrad_ok(s) && g.func == smallc::wgrad_fn(s)) {
    const float* x = (const float*)a[0]; const float* dy = (const float*)a[1]; float* dw = (float*)a[2];
    unsigned char* ws = (unsigned char*)a[14];
    switch (smallc::wg_nr(s)) {
      case 8: smallc::conv_wgrad_smallc_kernel<8><<<g.grid, g.block, g.smem, st>>>(x, dy, dw, s, ws, sig); break;
      case 9: smallc::conv_wgrad_smallc_kernel<9><<<g.grid, g.block, g.smem, st>>>(x, dy, dw, s, ws, sig); break;
      default: smallc::conv_wgrad_smallc_kernel<10><<<g.grid, g.block, g.smem, st>>>(x, dy, dw, s, ws, sig); break;
    }
    return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA;
  }
  long long M = s.K, N = (long long)s.R * s.S * s.C, K = (long long)s.N * s.P * s.Q;
  // A(m = kout, k = npq) = dy[npq * K + kout]
  return launch_tiled(g, M, N, K, (float*)a[2], N, nullptr, (float*)a[14], ADenseT{(const float*)a[1], s.K},
                      BWgrad{(const float*)a[0], s}, sig, st);
}
