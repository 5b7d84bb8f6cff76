// BatchNorm2d (NHWC, per-channel over rows = N*H*W): eval affine, train statistics with running-stat
// update, train apply, backward reduce and backward dx. Table 2 of the paper uses BN2d as the
// canonical memory-bound kernel. Reductions accumulate in fp64 per thread, combine
// row-lanes in a fixed order in shared memory, write per-split partials and let the last CTA of
// each channel block sum the splits in split order: deterministic, partition-independent.
#include "common.cuh"

namespace {

constexpr int BN_THREADS = 256;

// Channel block / row-lane split of a CTA for C channels.
__host__ __device__ inline int bn_cb(int C) { return C >= 64 ? 64 : (C >= 32 ? 32 : (C >= 16 ? 16 : (C >= 8 ? 8 : 4))); }

struct BnSplit { int cb, cblocks, rs; long long rows_per_split; };

BnSplit bn_split(long long rows, int C) {
  BnSplit s;
  s.cb = bn_cb(C);
  s.cblocks = (int)cdiv(C, s.cb);
  long long rs = cdiv(296, s.cblocks);               // shape-only: ~2 waves of a 148-SM part
  long long max_rs = cdiv(rows, 512);                  // >= 512 rows per split
  if (rs > max_rs) rs = max_rs;
  if (rs < 1) rs = 1;
  if (rs > 1024) rs = 1024;
  s.rs = (int)rs;
  s.rows_per_split = cdiv(rows, rs);
  return s;
}

uint64_t bn_ws_bytes(long long rows, int C, int nvals) {
  BnSplit s = bn_split(rows, C);
  return WS_TICKET_BYTES + (uint64_t)s.rs * C * nvals * 8;
}

// Reduce per-thread double accumulators v[NV] over the row-lanes of the CTA (fixed order) and
// write the CTA's partial for its channels to ws; returns true in the last CTA of the channel
// block, which must then combine partials (split order) via `combine`.
template <int NV>
__device__ bool bn_partial(double (&v)[NV], int C, int cb, int c0, int rs_count, unsigned char* ws, double* sh) {
  const int tid = threadIdx.x, rl_n = BN_THREADS / cb, cl = tid % cb, rl = tid / cb;
  // sh: [rl_n][cb][NV]
  for (int j = 0; j < NV; j++) sh[(rl * cb + cl) * NV + j] = v[j];
  __syncthreads();
  unsigned int* tickets = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  if (rl == 0) {
    double t[NV];
    for (int j = 0; j < NV; j++) t[j] = 0.0;
    for (int r = 0; r < rl_n; r++)
      for (int j = 0; j < NV; j++) t[j] += sh[(r * cb + cl) * NV + j];
    int c = c0 + cl;
    if (c < C)
      for (int j = 0; j < NV; j++) part[((long long)blockIdx.y * C + c) * NV + j] = t[j];
  }
  return last_cta_of(tickets + blockIdx.x, rs_count);
}

template <int NV>
__device__ void bn_combine(double (&t)[NV], int C, int c, int rs_count, unsigned char* ws, int cb) {
  (void)cb;
  const double* part = reinterpret_cast<const double*>(ws + WS_TICKET_BYTES);
  for (int j = 0; j < NV; j++) t[j] = 0.0;
  for (int r = 0; r < rs_count; r++)
    for (int j = 0; j < NV; j++) t[j] += __ldcg(part + ((long long)r * C + c) * NV + j);
}

// ---- train statistics: mean, invstd (biased var), running stats (unbiased var, momentum)
__global__ void __launch_bounds__(BN_THREADS) bn_stats_kernel(const float* __restrict__ x, float* mean, float* invstd, float* rm, float* rv,
                                                              long long rows, int C, float eps, float momentum, int cb,
                                                              long long rows_per_split, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[BN_THREADS * 2];
  const int rl_n = BN_THREADS / cb, cl = threadIdx.x % cb, rl = threadIdx.x / cb;
  const int c0 = blockIdx.x * cb, c = c0 + cl;
  const long long r0 = blockIdx.y * rows_per_split, r1 = min(rows, r0 + rows_per_split);
  double v[2] = {0.0, 0.0};
  if (c < C)
    for (long long r = r0 + rl; r < r1; r += rl_n) {
      double xv = (double)__ldg(x + r * C + c);
      v[0] += xv;
      v[1] += xv * xv;
    }
  if (bn_partial<2>(v, C, cb, c0, gridDim.y, ws, sh)) {
    if (rl == 0 && c < C) {
      double t[2];
      bn_combine<2>(t, C, c, gridDim.y, ws, cb);
      double m = t[0] / (double)rows;
      double var = t[1] / (double)rows - m * m;
      if (var < 0) var = 0;
      mean[c] = (float)m;
      invstd[c] = (float)(1.0 / sqrt(var + (double)eps));
      double unb = rows > 1 ? var * (double)rows / (double)(rows - 1) : var;
      rm[c] = (float)((1.0 - momentum) * (double)rm[c] + momentum * m);
      rv[c] = (float)((1.0 - momentum) * (double)rv[c] + momentum * unb);
    }
  }
  orion_signal(sig);
}

// ---- backward reduce: dbeta = sum dy, dgamma = sum dy * (x - mean) * invstd
__global__ void __launch_bounds__(BN_THREADS) bn_bwd_reduce_kernel(const float* __restrict__ x, const float* __restrict__ dy,
                                                                   const float* __restrict__ mean, const float* __restrict__ invstd,
                                                                   float* dgamma, float* dbeta, long long rows, int C, int cb,
                                                                   long long rows_per_split, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[BN_THREADS * 2];
  const int rl_n = BN_THREADS / cb, cl = threadIdx.x % cb, rl = threadIdx.x / cb;
  const int c0 = blockIdx.x * cb, c = c0 + cl;
  const long long r0 = blockIdx.y * rows_per_split, r1 = min(rows, r0 + rows_per_split);
  double v[2] = {0.0, 0.0};
  if (c < C) {
    const double mu = mean[c], is = invstd[c];
    for (long long r = r0 + rl; r < r1; r += rl_n) {
      double g = (double)__ldg(dy + r * C + c);
      double xh = ((double)__ldg(x + r * C + c) - mu) * is;
      v[0] += g;
      v[1] += g * xh;
    }
  }
  if (bn_partial<2>(v, C, cb, c0, gridDim.y, ws, sh)) {
    if (rl == 0 && c < C) {
      double t[2];
      bn_combine<2>(t, C, c, gridDim.y, ws, cb);
      dbeta[c] = (float)t[0];
      dgamma[c] = (float)t[1];
    }
  }
  orion_signal(sig);
}

// ---- elementwise per-channel affine kernels, float4 over channels (C % 4 == 0 on this path)
__global__ void __launch_bounds__(BN_THREADS) bn_eval_kernel(const float* __restrict__ x, float* __restrict__ y, const float* __restrict__ gamma,
                                                             const float* __restrict__ beta, const float* __restrict__ rm,
                                                             const float* __restrict__ rv, long long total, int C, float eps, OrionSig sig) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c = (int)(i % C);
    float sc = gamma[c] * rsqrtf(rv[c] + eps);
    y[i] = fmaf(x[i] - rm[c], sc, beta[c]);
  }
  orion_signal(sig);
}

__global__ void __launch_bounds__(BN_THREADS) bn_apply_kernel(const float* __restrict__ x, float* __restrict__ y, const float* __restrict__ gamma,
                                                              const float* __restrict__ beta, const float* __restrict__ mean,
                                                              const float* __restrict__ invstd, long long total, int C, OrionSig sig) {
  if ((C & 3) == 0) {
    long long nv = total / 4;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nv; i += (long long)gridDim.x * blockDim.x) {
      int c = (int)((i * 4) % C);
      float4 xv = __ldg(reinterpret_cast<const float4*>(x) + i);
      float4 m = __ldg(reinterpret_cast<const float4*>(mean + c));
      float4 is = __ldg(reinterpret_cast<const float4*>(invstd + c));
      float4 g = __ldg(reinterpret_cast<const float4*>(gamma + c));
      float4 b = __ldg(reinterpret_cast<const float4*>(beta + c));
      float4 o;
      o.x = fmaf(xv.x - m.x, is.x * g.x, b.x);
      o.y = fmaf(xv.y - m.y, is.y * g.y, b.y);
      o.z = fmaf(xv.z - m.z, is.z * g.z, b.z);
      o.w = fmaf(xv.w - m.w, is.w * g.w, b.w);
      reinterpret_cast<float4*>(y)[i] = o;
    }
  } else {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
      int c = (int)(i % C);
      y[i] = fmaf(x[i] - mean[c], invstd[c] * gamma[c], beta[c]);
    }
  }
  orion_signal(sig);
}

// dx = gamma*invstd/N * (N dy - dbeta - xhat dgamma)
__global__ void __launch_bounds__(BN_THREADS) bn_bwd_dx_kernel(const float* __restrict__ x, const float* __restrict__ dy, float* __restrict__ dx,
                                                               const float* __restrict__ gamma, const float* __restrict__ mean,
                                                               const float* __restrict__ invstd, const float* __restrict__ dgamma,
                                                               const float* __restrict__ dbeta, long long rows, int C, OrionSig sig) {
  // fp64 per element: dy and (dbeta + xhat*dgamma)/N nearly cancel, and fp32 would amplify the
  // rounding of each term through every BN layer of the backward pass (memory-bound: free)
  const long long total = rows * C;
  const double invN = 1.0 / (double)rows;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c = (int)(i % C);
    double is = invstd[c];
    double xh = ((double)x[i] - (double)mean[c]) * is;
    double k = (double)gamma[c] * is;
    dx[i] = (float)(k * ((double)dy[i] - ((double)dbeta[c] + xh * (double)dgamma[c]) * invN));
  }
  orion_signal(sig);
}

void ew(LaunchGeom* g, uint64_t n, const void* f) {
  uint64_t ctas = cdiv(n ? n : 1, BN_THREADS);
  if (ctas > 148 * 8) ctas = 148 * 8;
  g->grid = dim3((unsigned)ctas); g->block = dim3(BN_THREADS); g->smem = 0; g->func = f;
}

}  // namespace

extern "C" uint64_t orion_bn_workspace_bytes(uint64_t rows, uint64_t C) { return bn_ws_bytes((long long)rows, (int)C, 2); }

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

// BN eval: x, y, gamma, beta, rm, rv, rows, C, eps_bits
int bn_eval_geom(const uint64_t* a, LaunchGeom* g) { ew(g, a[6] * a[7], (const void*)bn_eval_kernel); return 0; }
int bn_eval_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  bn_eval_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (const float*)a[2], (const float*)a[3], (const float*)a[4],
                                            (const float*)a[5], (long long)(a[6] * a[7]), (int)a[7], u2f(a[8]), sig);
  CHECK_LAUNCH();
}

// BN stats: x, mean, invstd, rm, rv, rows, C, eps_bits, momentum_bits, ws, ws_bytes
int bn_stats_geom(const uint64_t* a, LaunchGeom* g) {
  if (a[9] == 0 || a[10] < bn_ws_bytes((long long)a[5], (int)a[6], 2)) return ORION_E_INVAL;
  BnSplit sp = bn_split((long long)a[5], (int)a[6]);
  g->grid = dim3(sp.cblocks, sp.rs); g->block = dim3(BN_THREADS); g->smem = 0; g->func = (const void*)bn_stats_kernel;
  return 0;
}
int bn_stats_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  BnSplit sp = bn_split((long long)a[5], (int)a[6]);
  bn_stats_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (float*)a[2], (float*)a[3], (float*)a[4], (long long)a[5],
                                             (int)a[6], u2f(a[7]), u2f(a[8]), sp.cb, sp.rows_per_split, (unsigned char*)a[9], sig);
  CHECK_LAUNCH();
}

// BN apply: x, y, gamma, beta, mean, invstd, rows, C
int bn_apply_geom(const uint64_t* a, LaunchGeom* g) { ew(g, (a[7] & 3) == 0 ? a[6] * a[7] / 4 : a[6] * a[7], (const void*)bn_apply_kernel); return 0; }
int bn_apply_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  bn_apply_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (const float*)a[2], (const float*)a[3], (const float*)a[4],
                                             (const float*)a[5], (long long)(a[6] * a[7]), (int)a[7], sig);
  CHECK_LAUNCH();
}

// BN bwd reduce: x, dy, mean, invstd, dgamma, dbeta, rows, C, ws, ws_bytes
int bn_bwd_reduce_geom(const uint64_t* a, LaunchGeom* g) {
  if (a[8] == 0 || a[9] < bn_ws_bytes((long long)a[6], (int)a[7], 2)) return ORION_E_INVAL;
  BnSplit sp = bn_split((long long)a[6], (int)a[7]);
  g->grid = dim3(sp.cblocks, sp.rs); g->block = dim3(BN_THREADS); g->smem = 0; g->func = (const void*)bn_bwd_reduce_kernel;
  return 0;
}
int bn_bwd_reduce_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  BnSplit sp = bn_split((long long)a[6], (int)a[7]);
  bn_bwd_reduce_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (const float*)a[2], (const float*)a[3],
                                                  (float*)a[4], (float*)a[5], (long long)a[6], (int)a[7], sp.cb, sp.rows_per_split,
                                                  (unsigned char*)a[8], sig);
  CHECK_LAUNCH();
}

// BN bwd dx: x, dy, dx, gamma, mean, invstd, dgamma, dbeta, rows, C
int bn_bwd_dx_geom(const uint64_t* a, LaunchGeom* g) { ew(g, a[8] * a[9], (const void*)bn_bwd_dx_kernel); return 0; }
int bn_bwd_dx_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  bn_bwd_dx_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (float*)a[2], (const float*)a[3], (const float*)a[4],
                                              (const float*)a[5], (const float*)a[6], (const float*)a[7], (long long)a[8], (int)a[9], sig);
  CHECK_LAUNCH();
}
