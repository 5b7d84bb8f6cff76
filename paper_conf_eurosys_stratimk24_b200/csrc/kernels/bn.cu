// BatchNorm2d (NHWC, per-channel over rows = N*H*W): eval affine, train statistics with running-stat
// update, train apply, backward reduce and backward dx. Table 2 of the paper uses BN2d as the
// canonical memory-bound kernel. Reductions accumulate in fp64 per thread, combine
// row-lanes in a fixed order in shared memory, write per-split partials and let the last CTA of
// each channel block sum the splits in split order: deterministic, partition-independent.
#include <cstdlib>

#include "common.cuh"

namespace {

constexpr int BN_THREADS = 256;

// Reduction kernels (train statistics, backward reduce). A thread owns 4 consecutive channels
// (128-bit loads; C % 4 == 0 on every BN of the workloads, checked at geometry time) and a
// row lane; a CTA owns CG4 channel quads x RL row lanes (RL*CG4 <= 256) and one row split. Rows
// are unrolled by 4 so each thread keeps 4 (stats) or 8 (backward) 128-bit loads in flight.
// fp64 accumulation, fixed-order combine of row lanes in smem, per-split partials combined in
// split order by the last CTA of the channel block.
struct BnSplit { int cg4, rl, cblocks, rs; long long rows_per_split; };

BnSplit bn_split(long long rows, int C) {
  BnSplit s;
  int q = C / 4;
  s.cg4 = q < 64 ? q : 64;
  s.rl = BN_THREADS / s.cg4;
  s.cblocks = (int)cdiv(q, s.cg4);
  // ~2 CTAs per SM: measured best over MobileNetV2's 12 BN shapes (tools/bench_kernels.py bn: 741 us
  // vs 830 at 4 per SM, 886 at 1 per SM for the stats + backward-reduce pairs)
  static const long long cta_target = getenv("ORION_BN_CTAS") ? atoll(getenv("ORION_BN_CTAS")) : 148 * 2;   // tuning knob
  static const long long min_rows = getenv("ORION_BN_MINROWS") ? atoll(getenv("ORION_BN_MINROWS")) : 16;
  long long rs = cdiv(cta_target, s.cblocks);   // shape-only (a 148-SM constant, not the partition)
  long long max_rs = cdiv(rows, min_rows * s.rl);   // >= 16 rows per row lane (2 trips of 8 loads)
  if (rs > max_rs) rs = max_rs;
  if (rs < 1) rs = 1;
  if (rs > 1024) rs = 1024;
  s.rs = (int)rs;
  s.rows_per_split = cdiv(rows, rs);
  return s;
}

// workspace: [tickets][split partials rs x C x nvals][group partials combine_rows(rs) x C x nvals]
uint64_t bn_ws_bytes(long long rows, int C, int nvals) {
  BnSplit s = bn_split(rows, C);
  return WS_TICKET_BYTES + (uint64_t)(s.rs + combine_rows(s.rs)) * C * nvals * 8;
}

struct D4 { double x, y, z, w; };
__device__ __forceinline__ void add4(D4& a, const float4& v) { a.x += v.x; a.y += v.y; a.z += v.z; a.w += v.w; }
__device__ __forceinline__ void sq4(D4& a, const float4& v) {
  a.x = fma((double)v.x, (double)v.x, a.x); a.y = fma((double)v.y, (double)v.y, a.y);
  a.z = fma((double)v.z, (double)v.z, a.z); a.w = fma((double)v.w, (double)v.w, a.w);
}

// Combine two D4 accumulators per thread over the CTA's row lanes (fixed order), write this
// split's partial for the CTA's channels, then combine the splits of the channel block in order
// (combine_splits). Returns true in the one CTA per channel block whose tot[(ch*2) + {0,1}]
// (ch = channel within the block) holds the totals.
__device__ bool bn_partial2(const D4& a, const D4& b, int C, int cg4, int rl_n, unsigned char* ws, double* sh, double* tot) {
  const int tid = threadIdx.x, cq = tid % cg4, rl = tid / cg4;
  const bool active = rl < rl_n;
  if (active) {
    double* d = sh + (size_t)(rl * cg4 + cq) * 8;
    d[0] = a.x; d[1] = a.y; d[2] = a.z; d[3] = a.w; d[4] = b.x; d[5] = b.y; d[6] = b.z; d[7] = b.w;
  }
  __syncthreads();
  unsigned int* tickets = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  const int c = (blockIdx.x * cg4 + cq) * 4;
  if (rl == 0 && c < C) {
    double t[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int r = 0; r < rl_n; r++)
      for (int j = 0; j < 8; j++) t[j] += sh[(size_t)(r * cg4 + cq) * 8 + j];
    for (int k = 0; k < 4; k++) {
      part[((long long)blockIdx.y * C + c + k) * 2 + 0] = t[k];
      part[((long long)blockIdx.y * C + c + k) * 2 + 1] = t[4 + k];
    }
  }
  const int rs = gridDim.y, cb0 = blockIdx.x * cg4 * 4;
  const int V = 2 * min(4 * cg4, C - cb0);
  return combine_splits(tickets + blockIdx.x * (combine_rows(rs) + 1), part + 2LL * cb0, part + 2LL * rs * C + 2LL * cb0, 2LL * C, rs,
                        blockIdx.y, V, tot, sh);
}

// ---- train statistics: mean, invstd (biased var), running stats (unbiased var, momentum)
__global__ void __launch_bounds__(BN_THREADS) bn_stats_kernel(const float* __restrict__ x, float* mean, float* invstd, float* rm, float* rv,
                                                              long long rows, int C, float eps, float momentum, int cg4, int rl_n,
                                                              long long rows_per_split, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[BN_THREADS * 8];
  const int cq = threadIdx.x % cg4, rl = threadIdx.x / cg4;
  const int c = (blockIdx.x * cg4 + cq) * 4;
  const long long r0 = blockIdx.y * rows_per_split, r1 = min(rows, r0 + rows_per_split);
  D4 s1{0, 0, 0, 0}, s2{0, 0, 0, 0};
  if (c < C && rl < rl_n) {
    const float* xp = x + c;
    long long r = r0 + rl;
    for (; r + 7LL * rl_n < r1; r += 8LL * rl_n) {
      float4 v[8];
#pragma unroll
      for (int i = 0; i < 8; i++) v[i] = __ldg(reinterpret_cast<const float4*>(xp + (r + i * (long long)rl_n) * C));
#pragma unroll
      for (int i = 0; i < 8; i++) { add4(s1, v[i]); sq4(s2, v[i]); }
    }
    for (; r < r1; r += rl_n) {
      float4 v = __ldg(reinterpret_cast<const float4*>(xp + r * C));
      add4(s1, v); sq4(s2, v);
    }
  }
  __shared__ double tot[BN_THREADS * 2];
  if (bn_partial2(s1, s2, C, cg4, rl_n, ws, sh, tot)) {
    if (rl == 0 && c < C) {
      for (int k = 0; k < 4; k++) {
        double t0 = tot[(cq * 4 + k) * 2], t1 = tot[(cq * 4 + k) * 2 + 1];
        double m = t0 / (double)rows;
        double var = t1 / (double)rows - m * m;
        if (var < 0) var = 0;
        mean[c + k] = (float)m;
        invstd[c + k] = (float)(1.0 / sqrt(var + (double)eps));
        double unb = rows > 1 ? var * (double)rows / (double)(rows - 1) : var;
        rm[c + k] = (float)((1.0 - momentum) * (double)rm[c + k] + momentum * m);
        rv[c + k] = (float)((1.0 - momentum) * (double)rv[c + k] + momentum * unb);
      }
    }
  }
  orion_signal(sig);
}

// ---- backward reduce: dbeta = sum dy, dgamma = sum dy * (x - mean) * invstd
__global__ void __launch_bounds__(BN_THREADS) bn_bwd_reduce_kernel(const float* __restrict__ x, const float* __restrict__ dy,
                                                                   const float* __restrict__ mean, const float* __restrict__ invstd,
                                                                   float* dgamma, float* dbeta, long long rows, int C, int cg4, int rl_n,
                                                                   long long rows_per_split, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[BN_THREADS * 8];
  const int cq = threadIdx.x % cg4, rl = threadIdx.x / cg4;
  const int c = (blockIdx.x * cg4 + cq) * 4;
  const long long r0 = blockIdx.y * rows_per_split, r1 = min(rows, r0 + rows_per_split);
  // sum dy (x - mean) invstd = invstd (sum dy x - mean sum dy): accumulate sum dy and sum dy x
  // (the fp32 product is exact in fp64), so an element costs 2 conversions, 1 DADD and 1 DFMA;
  // the last CTA of the channel block applies mean and invstd once
  D4 sg{0, 0, 0, 0}, sgx{0, 0, 0, 0};
  if (c < C && rl < rl_n) {
    const float* xp = x + c;
    const float* gp = dy + c;
    auto acc = [&](const float4& g, const float4& v) {
      sg.x += g.x; sg.y += g.y; sg.z += g.z; sg.w += g.w;
      sgx.x = fma((double)g.x, (double)v.x, sgx.x);
      sgx.y = fma((double)g.y, (double)v.y, sgx.y);
      sgx.z = fma((double)g.z, (double)v.z, sgx.z);
      sgx.w = fma((double)g.w, (double)v.w, sgx.w);
    };
    long long r = r0 + rl;
    for (; r + 3LL * rl_n < r1; r += 4LL * rl_n) {
      float4 g0 = __ldg(reinterpret_cast<const float4*>(gp + r * C));
      float4 g1 = __ldg(reinterpret_cast<const float4*>(gp + (r + rl_n) * C));
      float4 g2 = __ldg(reinterpret_cast<const float4*>(gp + (r + 2LL * rl_n) * C));
      float4 g3 = __ldg(reinterpret_cast<const float4*>(gp + (r + 3LL * rl_n) * C));
      float4 v0 = __ldg(reinterpret_cast<const float4*>(xp + r * C));
      float4 v1 = __ldg(reinterpret_cast<const float4*>(xp + (r + rl_n) * C));
      float4 v2 = __ldg(reinterpret_cast<const float4*>(xp + (r + 2LL * rl_n) * C));
      float4 v3 = __ldg(reinterpret_cast<const float4*>(xp + (r + 3LL * rl_n) * C));
      acc(g0, v0); acc(g1, v1); acc(g2, v2); acc(g3, v3);
    }
    for (; r < r1; r += rl_n)
      acc(__ldg(reinterpret_cast<const float4*>(gp + r * C)), __ldg(reinterpret_cast<const float4*>(xp + r * C)));
  }
  __shared__ double tot[BN_THREADS * 2];
  if (bn_partial2(sg, sgx, C, cg4, rl_n, ws, sh, tot)) {
    if (rl == 0 && c < C) {
      for (int k = 0; k < 4; k++) {
        double t0 = tot[(cq * 4 + k) * 2], t1 = tot[(cq * 4 + k) * 2 + 1];
        dbeta[c + k] = (float)t0;
        dgamma[c + k] = (float)((double)invstd[c + k] * (t1 - (double)mean[c + k] * t0));
      }
    }
  }
  orion_signal(sig);
}

// ---- elementwise per-channel affine kernels, float4 over channels (C % 4 == 0 on this path)
__global__ void __launch_bounds__(BN_THREADS) bn_eval_kernel(const float* __restrict__ x, float* __restrict__ y, const float* __restrict__ gamma,
                                                             const float* __restrict__ beta, const float* __restrict__ rm,
                                                             const float* __restrict__ rv, long long total, int C, float eps, OrionSig sig) {
  if ((C & 3) == 0) {
    // fixed channel quad per thread: the per-channel scale g * rsqrt(var + eps) (the same fp32
    // operations as the scalar path, so bit-identical to it) is formed once, lanes stride over rows
    const int q = C / 4;
    const long long rows = total / C;
    const long long gt = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long L = ((long long)gridDim.x * blockDim.x) / q;
    const int cq = (int)(gt % q);
    const long long lane = gt / q;
    if (lane < L) {
      const int c = cq * 4;
      const float4 g = __ldg(reinterpret_cast<const float4*>(gamma + c)), b = __ldg(reinterpret_cast<const float4*>(beta + c));
      const float4 m = __ldg(reinterpret_cast<const float4*>(rm + c)), v = __ldg(reinterpret_cast<const float4*>(rv + c));
      const float4 sc = make_float4(g.x * rsqrtf(v.x + eps), g.y * rsqrtf(v.y + eps), g.z * rsqrtf(v.z + eps), g.w * rsqrtf(v.w + eps));
      auto one = [&](const float4& xv) {
        return make_float4(fmaf(xv.x - m.x, sc.x, b.x), fmaf(xv.y - m.y, sc.y, b.y), fmaf(xv.z - m.z, sc.z, b.z), fmaf(xv.w - m.w, sc.w, b.w));
      };
      const float4* x4 = reinterpret_cast<const float4*>(x);
      float4* y4 = reinterpret_cast<float4*>(y);
      long long r = lane;
      for (; r + 3 * L < rows; r += 4 * L) {
        const long long i0 = r * q + cq, i1 = (r + L) * q + cq, i2 = (r + 2 * L) * q + cq, i3 = (r + 3 * L) * q + cq;
        const float4 a0 = __ldg(x4 + i0), a1 = __ldg(x4 + i1), a2 = __ldg(x4 + i2), a3 = __ldg(x4 + i3);
        y4[i0] = one(a0); y4[i1] = one(a1); y4[i2] = one(a2); y4[i3] = one(a3);
      }
      for (; r < rows; r += L) y4[r * q + cq] = one(__ldg(x4 + r * q + cq));
    }
  } else {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
      int c = (int)(i % C);
      float sc = gamma[c] * rsqrtf(rv[c] + eps);
      y[i] = fmaf(x[i] - rm[c], sc, beta[c]);
    }
  }
  orion_signal(sig);
}

__global__ void __launch_bounds__(BN_THREADS) bn_apply_kernel(const float* __restrict__ x, float* __restrict__ y, const float* __restrict__ gamma,
                                                              const float* __restrict__ beta, const float* __restrict__ mean,
                                                              const float* __restrict__ invstd, long long total, int C, OrionSig sig) {
  if ((C & 3) == 0) {
    // fixed channel quad per thread (per-channel vectors loaded once), lanes stride over rows
    const int q = C / 4;
    const long long rows = total / C;
    const long long gt = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long L = ((long long)gridDim.x * blockDim.x) / q;
    const int cq = (int)(gt % q);
    const long long lane = gt / q;
    if (lane < L) {
      const int c = cq * 4;
      const float4 m = __ldg(reinterpret_cast<const float4*>(mean + c));
      const float4 is = __ldg(reinterpret_cast<const float4*>(invstd + c));
      const float4 g = __ldg(reinterpret_cast<const float4*>(gamma + c));
      const float4 b = __ldg(reinterpret_cast<const float4*>(beta + c));
      const float4 sc = make_float4(is.x * g.x, is.y * g.y, is.z * g.z, is.w * g.w);
      auto one = [&](const float4& xv) {
        return make_float4(fmaf(xv.x - m.x, sc.x, b.x), fmaf(xv.y - m.y, sc.y, b.y), fmaf(xv.z - m.z, sc.z, b.z), fmaf(xv.w - m.w, sc.w, b.w));
      };
      const float4* x4 = reinterpret_cast<const float4*>(x);
      float4* y4 = reinterpret_cast<float4*>(y);
      long long r = lane;
      for (; r + 3 * L < rows; r += 4 * L) {
        const long long i0 = r * q + cq, i1 = (r + L) * q + cq, i2 = (r + 2 * L) * q + cq, i3 = (r + 3 * L) * q + cq;
        const float4 a0 = __ldg(x4 + i0), a1 = __ldg(x4 + i1), a2 = __ldg(x4 + i2), a3 = __ldg(x4 + i3);
        y4[i0] = one(a0); y4[i1] = one(a1); y4[i2] = one(a2); y4[i3] = one(a3);
      }
      for (; r < rows; r += L) y4[r * q + cq] = one(__ldg(x4 + r * q + cq));
    }
  } else {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
      int c = (int)(i % C);
      y[i] = fmaf(x[i] - mean[c], invstd[c] * gamma[c], beta[c]);
    }
  }
  orion_signal(sig);
}

// dx = gamma*invstd/N (N dy - dbeta - xhat dgamma), evaluated in fp64 per element: dy and
// (dbeta + xhat*dgamma)/N nearly cancel, and fp32 would amplify the rounding of each term through
// every BN layer of the backward pass (memory-bound kernel: the fp64 math is free).
__device__ __forceinline__ float bn_dx1(float x, float dy, float g, float m, float is, float dg, float db, double invN) {
  double xh = ((double)x - (double)m) * (double)is;
  return (float)((double)g * (double)is * ((double)dy - ((double)db + xh * (double)dg) * invN));
}
__global__ void __launch_bounds__(BN_THREADS) bn_bwd_dx_kernel(const float* __restrict__ x, const float* __restrict__ dy, float* __restrict__ dx,
                                                               const float* __restrict__ gamma, const float* __restrict__ mean,
                                                               const float* __restrict__ invstd, const float* __restrict__ dgamma,
                                                               const float* __restrict__ dbeta, long long rows, int C, OrionSig sig) {
  const long long total = rows * C;
  const double invN = 1.0 / (double)rows;
  if ((C & 3) == 0) {
    // thread -> fixed channel quad cq (its 5 per-channel vectors loaded once) and row lane; lanes
    // stride over rows, so a warp's 32 float4 loads are consecutive in memory; 2 rows in flight
    const int q = C / 4;
    const long long gt = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long L = ((long long)gridDim.x * blockDim.x) / q;
    const int cq = (int)(gt % q);
    const long long lane = gt / q;
    if (lane < L) {
      const int c = cq * 4;
      // dx = A dy + B x + K per channel, A = gamma invstd, B = -A invstd dgamma / N,
      // K = -A dbeta / N - B mean (the expression above expanded; coefficients in fp64 once per
      // thread, so an element costs 2 conversions in, 2 DFMA and 1 conversion out)
      double A[4], B[4], K[4];
      {
        const float4 ga = __ldg(reinterpret_cast<const float4*>(gamma + c)), mu = __ldg(reinterpret_cast<const float4*>(mean + c));
        const float4 is = __ldg(reinterpret_cast<const float4*>(invstd + c)), dg = __ldg(reinterpret_cast<const float4*>(dgamma + c));
        const float4 db = __ldg(reinterpret_cast<const float4*>(dbeta + c));
        const float gv[4] = {ga.x, ga.y, ga.z, ga.w}, mv[4] = {mu.x, mu.y, mu.z, mu.w}, iv[4] = {is.x, is.y, is.z, is.w};
        const float dgv[4] = {dg.x, dg.y, dg.z, dg.w}, dbv[4] = {db.x, db.y, db.z, db.w};
#pragma unroll
        for (int k = 0; k < 4; k++) {
          A[k] = (double)gv[k] * (double)iv[k];
          B[k] = -A[k] * (double)iv[k] * (double)dgv[k] * invN;
          K[k] = -A[k] * (double)dbv[k] * invN - B[k] * (double)mv[k];
        }
      }
      auto one = [&](const float4& xv, const float4& gv) {
        float4 o;
        o.x = (float)fma(A[0], (double)gv.x, fma(B[0], (double)xv.x, K[0]));
        o.y = (float)fma(A[1], (double)gv.y, fma(B[1], (double)xv.y, K[1]));
        o.z = (float)fma(A[2], (double)gv.z, fma(B[2], (double)xv.z, K[2]));
        o.w = (float)fma(A[3], (double)gv.w, fma(B[3], (double)xv.w, K[3]));
        return o;
      };
      const float4* x4 = reinterpret_cast<const float4*>(x);
      const float4* g4 = reinterpret_cast<const float4*>(dy);
      float4* d4 = reinterpret_cast<float4*>(dx);
      long long r = lane;
      for (; r + L < rows; r += 2 * L) {
        const long long i0 = r * q + cq, i1 = (r + L) * q + cq;
        const float4 x0 = __ldg(x4 + i0), g0 = __ldg(g4 + i0), x1 = __ldg(x4 + i1), g1 = __ldg(g4 + i1);
        d4[i0] = one(x0, g0);
        d4[i1] = one(x1, g1);
      }
      if (r < rows) {
        const long long i0 = r * q + cq;
        d4[i0] = one(__ldg(x4 + i0), __ldg(g4 + i0));
      }
    }
  } else {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
      int c = (int)(i % C);
      dx[i] = bn_dx1(x[i], dy[i], gamma[c], mean[c], invstd[c], dgamma[c], dbeta[c], invN);
    }
  }
  orion_signal(sig);
}

void ew(LaunchGeom* g, uint64_t n, const void* f, std::atomic<int>& occ) {
  uint64_t ctas = cdiv(n ? n : 1, BN_THREADS);
  const uint64_t wave = 148ull * resident_ctas_per_sm(f, BN_THREADS, occ);
  if (ctas > wave) ctas = wave;
  g->grid = dim3((unsigned)ctas); g->block = dim3(BN_THREADS); g->smem = 0; g->func = f;
}

}  // namespace

extern "C" uint64_t orion_bn_workspace_bytes(uint64_t rows, uint64_t C) { return bn_ws_bytes((long long)rows, (int)C, 2); }

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

// BN eval: x, y, gamma, beta, rm, rv, rows, C, eps_bits
std::atomic<int> bn_eval_occ{0};
int bn_eval_geom(const uint64_t* a, LaunchGeom* g) { ew(g, (a[7] & 3) == 0 ? a[6] * a[7] / 4 : a[6] * a[7], (const void*)bn_eval_kernel, bn_eval_occ); return 0; }
int bn_eval_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  bn_eval_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (const float*)a[2], (const float*)a[3], (const float*)a[4],
                                            (const float*)a[5], (long long)(a[6] * a[7]), (int)a[7], u2f(a[8]), sig);
  CHECK_LAUNCH();
}

// BN stats: x, mean, invstd, rm, rv, rows, C, eps_bits, momentum_bits, ws, ws_bytes
int bn_stats_geom(const uint64_t* a, LaunchGeom* g) {
  if ((a[6] & 3) || a[9] == 0 || a[10] < bn_ws_bytes((long long)a[5], (int)a[6], 2)) return ORION_E_INVAL;
  BnSplit sp = bn_split((long long)a[5], (int)a[6]);
  g->grid = dim3(sp.cblocks, sp.rs); g->block = dim3(BN_THREADS); g->smem = 0; g->func = (const void*)bn_stats_kernel;
  return 0;
}
int bn_stats_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  BnSplit sp = bn_split((long long)a[5], (int)a[6]);
  bn_stats_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (float*)a[2], (float*)a[3], (float*)a[4], (long long)a[5],
                                             (int)a[6], u2f(a[7]), u2f(a[8]), sp.cg4, sp.rl, sp.rows_per_split, (unsigned char*)a[9], sig);
  CHECK_LAUNCH();
}

// BN apply: x, y, gamma, beta, mean, invstd, rows, C
std::atomic<int> bn_apply_occ{0};
int bn_apply_geom(const uint64_t* a, LaunchGeom* g) { ew(g, (a[7] & 3) == 0 ? a[6] * a[7] / 4 : a[6] * a[7], (const void*)bn_apply_kernel, bn_apply_occ); return 0; }
int bn_apply_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  bn_apply_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (const float*)a[2], (const float*)a[3], (const float*)a[4],
                                             (const float*)a[5], (long long)(a[6] * a[7]), (int)a[7], sig);
  CHECK_LAUNCH();
}

// BN bwd reduce: x, dy, mean, invstd, dgamma, dbeta, rows, C, ws, ws_bytes
int bn_bwd_reduce_geom(const uint64_t* a, LaunchGeom* g) {
  if ((a[7] & 3) || a[8] == 0 || a[9] < bn_ws_bytes((long long)a[6], (int)a[7], 2)) return ORION_E_INVAL;
  BnSplit sp = bn_split((long long)a[6], (int)a[7]);
  g->grid = dim3(sp.cblocks, sp.rs); g->block = dim3(BN_THREADS); g->smem = 0; g->func = (const void*)bn_bwd_reduce_kernel;
  return 0;
}
int bn_bwd_reduce_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  BnSplit sp = bn_split((long long)a[6], (int)a[7]);
  bn_bwd_reduce_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (const float*)a[2], (const float*)a[3],
                                                  (float*)a[4], (float*)a[5], (long long)a[6], (int)a[7], sp.cg4, sp.rl,
                                                  sp.rows_per_split, (unsigned char*)a[8], sig);
  CHECK_LAUNCH();
}

// BN bwd dx: x, dy, dx, gamma, mean, invstd, dgamma, dbeta, rows, C
std::atomic<int> bn_bwd_dx_occ{0};
int bn_bwd_dx_geom(const uint64_t* a, LaunchGeom* g) { ew(g, (a[9] & 3) == 0 ? a[8] * a[9] / 4 : a[8] * a[9], (const void*)bn_bwd_dx_kernel, bn_bwd_dx_occ); return 0; }
int bn_bwd_dx_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  bn_bwd_dx_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (float*)a[2], (const float*)a[3], (const float*)a[4],
                                              (const float*)a[5], (const float*)a[6], (const float*)a[7], (long long)a[8], (int)a[9], sig);
  CHECK_LAUNCH();
}
