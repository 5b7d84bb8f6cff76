// Memory-bound operators: activations, residual add, pooling, losses, SGD, bias-grad column sum.
// 128-bit vectorised grid-stride loops (HBM-bound; DESIGN.md §7 gives bytes per element);
// reductions use fixed-order warp-shuffle trees and last-CTA ordered finalisation (deterministic).
#include <float.h>
#include "common.cuh"

namespace {

constexpr int EW_THREADS = 256;
constexpr unsigned EW_MAX_CTAS = 148 * 8;  // shape-independent cap; results never depend on grid size

__host__ __device__ inline bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

void ew_geom(LaunchGeom* g, uint64_t n_vec, const void* f) {
  uint64_t ctas = cdiv(n_vec ? n_vec : 1, EW_THREADS);
  g->grid = dim3((unsigned)(ctas < EW_MAX_CTAS ? ctas : EW_MAX_CTAS));
  g->block = dim3(EW_THREADS);
  g->smem = 0;
  g->func = f;
}

template <class Op>
__global__ void __launch_bounds__(EW_THREADS) unary_kernel(const float* __restrict__ x, float* __restrict__ y, long long n, Op op, OrionSig sig) {
  long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  long long stride = (long long)gridDim.x * blockDim.x;
  if (aligned16(x) && aligned16(y)) {
    long long nv = n / 4;
    for (long long i = i0; i < nv; i += stride) {
      float4 v = __ldg(reinterpret_cast<const float4*>(x) + i);
      v.x = op(v.x); v.y = op(v.y); v.z = op(v.z); v.w = op(v.w);
      reinterpret_cast<float4*>(y)[i] = v;
    }
    for (long long i = nv * 4 + i0; i < n; i += stride) y[i] = op(x[i]);
  } else {
    for (long long i = i0; i < n; i += stride) y[i] = op(x[i]);
  }
  orion_signal(sig);
}

template <class Op>
__global__ void __launch_bounds__(EW_THREADS) binary_kernel(const float* __restrict__ a, const float* __restrict__ b, float* __restrict__ c,
                                                            long long n, Op op, OrionSig sig) {
  long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  long long stride = (long long)gridDim.x * blockDim.x;
  if (aligned16(a) && aligned16(b) && aligned16(c)) {
    long long nv = n / 4;
    for (long long i = i0; i < nv; i += stride) {
      float4 u = __ldg(reinterpret_cast<const float4*>(a) + i);
      float4 v = __ldg(reinterpret_cast<const float4*>(b) + i);
      float4 w;
      w.x = op(u.x, v.x); w.y = op(u.y, v.y); w.z = op(u.z, v.z); w.w = op(u.w, v.w);
      reinterpret_cast<float4*>(c)[i] = w;
    }
    for (long long i = nv * 4 + i0; i < n; i += stride) c[i] = op(a[i], b[i]);
  } else {
    for (long long i = i0; i < n; i += stride) c[i] = op(a[i], b[i]);
  }
  orion_signal(sig);
}

struct ReluOp { __device__ float operator()(float x) const { return x > 0.f ? x : 0.f; } };
struct Relu6Op { __device__ float operator()(float x) const { return fminf(fmaxf(x, 0.f), 6.f); } };
// binary ops take (x, dy) for the backward ones
struct ReluBwdOp { __device__ float operator()(float x, float dy) const { return x > 0.f ? dy : 0.f; } };
struct Relu6BwdOp { __device__ float operator()(float x, float dy) const { return (x > 0.f && x < 6.f) ? dy : 0.f; } };
struct AddOp { __device__ float operator()(float a, float b) const { return a + b; } };

// ---- SGD: v = mu v + g ; p -= lr v   (mu == 0: p -= lr g)
__global__ void __launch_bounds__(EW_THREADS) sgd_kernel(float* __restrict__ p, const float* __restrict__ g, float* __restrict__ v,
                                                         long long n, float lr, float mu, OrionSig sig) {
  long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = i0; i < n; i += stride) {
    float gi = g[i];
    if (mu != 0.f) {
      float vi = fmaf(mu, v[i], gi);
      v[i] = vi;
      p[i] = p[i] - lr * vi;
    } else {
      p[i] = p[i] - lr * gi;
    }
  }
  orion_signal(sig);
}

// ---- column sum (bias gradient): out[n] = sum_m A[m][n]. A CTA owns CS_COLS columns (8 column
// quads, 128-bit loads when N % 4 == 0) and all M rows, split over 32 row lanes: lane l sums rows
// l, l + 32, ... in fp32 (8 loads in flight), the lanes are added in lane order in fp64. One pass
// over A with N / CS_COLS CTAs (the round-1 thread-per-column loop ran 6 CTAs at ~56 GB/s);
// fixed order, no workspace, deterministic.
constexpr int CS_QUADS = 8, CS_LANES = EW_THREADS / CS_QUADS, CS_COLS = 4 * CS_QUADS;
__global__ void __launch_bounds__(EW_THREADS) colsum_kernel(const float* __restrict__ A, float* __restrict__ out, int M, int N, OrionSig sig) {
  __shared__ float4 part[CS_LANES][CS_QUADS];
  const int q = threadIdx.x % CS_QUADS, lane = threadIdx.x / CS_QUADS;
  const int n = blockIdx.x * CS_COLS + 4 * q;
  float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
  if (n < N) {
    const bool vec = (N % 4 == 0);
    auto ld = [&](long long m) -> float4 {
      const float* p = A + m * N + n;
      if (vec) return __ldg(reinterpret_cast<const float4*>(p));
      return make_float4(__ldg(p), n + 1 < N ? __ldg(p + 1) : 0.f, n + 2 < N ? __ldg(p + 2) : 0.f, n + 3 < N ? __ldg(p + 3) : 0.f);
    };
    int m = lane;
    for (; m + 7 * CS_LANES < M; m += 8 * CS_LANES) {
      float4 v[8];
#pragma unroll
      for (int i = 0; i < 8; i++) v[i] = ld(m + (long long)i * CS_LANES);
#pragma unroll
      for (int i = 0; i < 8; i++) { s.x += v[i].x; s.y += v[i].y; s.z += v[i].z; s.w += v[i].w; }
    }
    for (; m < M; m += CS_LANES) {
      const float4 v = ld(m);
      s.x += v.x; s.y += v.y; s.z += v.z; s.w += v.w;
    }
  }
  part[lane][q] = s;
  __syncthreads();
  if (threadIdx.x < CS_COLS) {
    const int qq = threadIdx.x / 4, j = threadIdx.x % 4, col = blockIdx.x * CS_COLS + threadIdx.x;
    double t = 0.0;
    for (int l = 0; l < CS_LANES; l++) {
      const float4 v = part[l][qq];
      t += (double)(j == 0 ? v.x : j == 1 ? v.y : j == 2 ? v.z : v.w);
    }
    if (col < N) out[col] = (float)t;
  }
  orion_signal(sig);
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
// fixed-order block reduction (all threads get the result)
template <bool kMax>
__device__ float block_reduce(float v, float* sh) {
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32, nw = blockDim.x / 32;
  v = kMax ? warp_max(v) : warp_sum(v);
  __syncthreads();
  if (lane == 0) sh[warp] = v;
  __syncthreads();
  float r = kMax ? -FLT_MAX : 0.f;
  if (warp == 0) {
    float t = lane < nw ? sh[lane] : (kMax ? -FLT_MAX : 0.f);
    r = kMax ? warp_max(t) : warp_sum(t);
    if (lane == 0) sh[0] = r;
  }
  __syncthreads();
  r = sh[0];
  __syncthreads();
  return r;
}
__device__ double block_reduce_d(double v, double* sh) {
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32, nw = blockDim.x / 32;
  v = warp_sum_d(v);
  __syncthreads();
  if (lane == 0) sh[warp] = v;
  __syncthreads();
  if (warp == 0) {
    double t = lane < nw ? sh[lane] : 0.0;
    t = warp_sum_d(t);
    if (lane == 0) sh[0] = t;
  }
  __syncthreads();
  double r = sh[0];
  __syncthreads();
  return r;
}

// ---- MSE: loss = mean((y-t)^2), dy = 2(y-t)/n. ws: [ticket u32 | pad][double partial per CTA]
__global__ void __launch_bounds__(EW_THREADS) mse_kernel(const float* __restrict__ y, const float* __restrict__ t, float* __restrict__ loss,
                                                         float* __restrict__ dy, long long n, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[32];
  unsigned int* ticket = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  long long stride = (long long)gridDim.x * blockDim.x;
  double acc = 0.0;
  const float scale = 2.0f / (float)n;
  for (long long i = i0; i < n; i += stride) {
    float d = y[i] - t[i];
    acc += (double)d * (double)d;
    dy[i] = scale * d;
  }
  double s = block_reduce_d(acc, sh);
  if (threadIdx.x == 0) part[blockIdx.x] = s;
  if (last_cta_of(ticket, gridDim.x)) {
    if (threadIdx.x == 0) {
      double tot = 0.0;
      for (unsigned b = 0; b < gridDim.x; b++) tot += __ldcg(part + b);
      *loss = (float)(tot / (double)n);
    }
  }
  orion_signal(sig);
}

// ---- softmax cross entropy, mean over batch. One CTA per row. ws: [ticket | pad][float row loss]
__global__ void __launch_bounds__(EW_THREADS) ce_kernel(const float* __restrict__ z, const int* __restrict__ labels, float* __restrict__ loss,
                                                        float* __restrict__ dz, int B, int Cn, unsigned char* ws, OrionSig sig) {
  __shared__ float sh[32];
  unsigned int* ticket = reinterpret_cast<unsigned int*>(ws);
  float* rowloss = reinterpret_cast<float*>(ws + WS_TICKET_BYTES);
  const int b = blockIdx.x;
  const float* zr = z + (long long)b * Cn;
  float m = -FLT_MAX;
  for (int c = threadIdx.x; c < Cn; c += blockDim.x) m = fmaxf(m, zr[c]);
  m = block_reduce<true>(m, sh);
  float s = 0.f;
  for (int c = threadIdx.x; c < Cn; c += blockDim.x) s += expf(zr[c] - m);
  s = block_reduce<false>(s, sh);
  const float lse = m + logf(s);
  const int y = labels[b];
  const float invB = 1.0f / (float)B;
  for (int c = threadIdx.x; c < Cn; c += blockDim.x) {
    float pc = expf(zr[c] - lse);
    dz[(long long)b * Cn + c] = (pc - (c == y ? 1.f : 0.f)) * invB;
  }
  if (threadIdx.x == 0) rowloss[b] = lse - zr[y];
  if (last_cta_of(ticket, gridDim.x)) {
    if (threadIdx.x == 0) {
      double tot = 0.0;
      for (int r = 0; r < B; r++) tot += (double)__ldcg(rowloss + r);
      *loss = (float)(tot / (double)B);
    }
  }
  orion_signal(sig);
}

// ---- MaxPool 3x3 / 2, pad 1 (-inf padding), NHWC, thread per output channel quad (128-bit loads;
// the workloads' C % 4 == 0, checked at geometry time); fmaxf per channel, as the scalar form
__global__ void __launch_bounds__(EW_THREADS) maxpool_kernel(const float* __restrict__ x, float* __restrict__ y, int N, int H, int W, int C,
                                                             int P, int Q, OrionSig sig) {
  const int C4 = C / 4;
  long long total = (long long)N * P * Q * C4;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c = (int)(i % C4) * 4; long long t = i / C4;
    int q = (int)(t % Q); t /= Q;
    int p = (int)(t % P); int n = (int)(t / P);
    float4 m = make_float4(-FLT_MAX, -FLT_MAX, -FLT_MAX, -FLT_MAX);
#pragma unroll
    for (int r = 0; r < 3; r++) {
      int h = 2 * p - 1 + r;
      if ((unsigned)h >= (unsigned)H) continue;
#pragma unroll
      for (int s = 0; s < 3; s++) {
        int w = 2 * q - 1 + s;
        if ((unsigned)w >= (unsigned)W) continue;
        const float4 v = __ldg(reinterpret_cast<const float4*>(x + (((long long)n * H + h) * W + w) * C + c));
        m.x = fmaxf(m.x, v.x); m.y = fmaxf(m.y, v.y); m.z = fmaxf(m.z, v.z); m.w = fmaxf(m.w, v.w);
      }
    }
    reinterpret_cast<float4*>(y)[i] = m;
  }
  orion_signal(sig);
}

// ---- global average pool [N, HW, C] -> [N, C], sequential over HW per (n, c)
__global__ void __launch_bounds__(EW_THREADS) avgpool_kernel(const float* __restrict__ x, float* __restrict__ y, int N, int HW, int C, OrionSig sig) {
  long long total = (long long)N * C;
  const float inv = 1.0f / (float)HW;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c = (int)(i % C); long long n = i / C;
    const float* xp = x + n * HW * C + c;
    float s = 0.f;
    for (int k = 0; k < HW; k++) s += __ldg(xp + (long long)k * C);
    y[i] = s * inv;
  }
  orion_signal(sig);
}

__global__ void __launch_bounds__(EW_THREADS) avgpool_bwd_kernel(const float* __restrict__ dy, float* __restrict__ dx, int N, int HW, int C, OrionSig sig) {
  long long total = (long long)N * HW * C;
  const float inv = 1.0f / (float)HW;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c = (int)(i % C); long long n = i / ((long long)HW * C);
    dx[i] = __ldg(dy + n * C + c) * inv;
  }
  orion_signal(sig);
}

}  // namespace

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

// ---- unary: args x, y, n
#define UNARY_ENTRY(name, Op)                                                                    \
  int name##_geom(const uint64_t* a, LaunchGeom* g) { ew_geom(g, cdiv(a[2], 4), (const void*)unary_kernel<Op>); return 0; } \
  int name##_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {    \
    unary_kernel<Op><<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (long long)a[2], Op{}, sig); \
    CHECK_LAUNCH(); }
UNARY_ENTRY(relu, ReluOp)
UNARY_ENTRY(relu6, Relu6Op)

// ---- binary: args a, b, c, n
#define BINARY_ENTRY(name, Op)                                                                   \
  int name##_geom(const uint64_t* a, LaunchGeom* g) { ew_geom(g, cdiv(a[3], 4), (const void*)binary_kernel<Op>); return 0; } \
  int name##_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {     \
    binary_kernel<Op><<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (float*)a[2], (long long)a[3], Op{}, sig); \
    CHECK_LAUNCH(); }
BINARY_ENTRY(relu_bwd, ReluBwdOp)
BINARY_ENTRY(relu6_bwd, Relu6BwdOp)
BINARY_ENTRY(add, AddOp)

// ---- SGD: args p, g, v, n, lr_bits, mu_bits
int sgd_geom(const uint64_t* a, LaunchGeom* g) { ew_geom(g, a[3], (const void*)sgd_kernel); return 0; }
int sgd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  sgd_kernel<<<g.grid, g.block, 0, s>>>((float*)a[0], (const float*)a[1], (float*)a[2], (long long)a[3], u2f(a[4]), u2f(a[5]), sig);
  CHECK_LAUNCH();
}

// ---- colsum: args A, out, M, N
int colsum_geom(const uint64_t* a, LaunchGeom* g) {
  g->grid = dim3((unsigned)cdiv(a[3], CS_COLS)); g->block = dim3(EW_THREADS); g->smem = 0; g->func = (const void*)colsum_kernel;
  return 0;
}
int colsum_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  colsum_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (int)a[2], (int)a[3], sig);
  CHECK_LAUNCH();
}

// ---- MSE: args y, t, loss, dy, n, ws (>= WS_TICKET_BYTES + 8 * ctas bytes, zeroed once)
int mse_geom(const uint64_t* a, LaunchGeom* g) { ew_geom(g, a[4], (const void*)mse_kernel); return 0; }
int mse_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  mse_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const float*)a[1], (float*)a[2], (float*)a[3], (long long)a[4],
                                        (unsigned char*)a[5], sig);
  CHECK_LAUNCH();
}

// ---- CE: args z, labels, loss, dz, B, classes, ws (>= WS_TICKET_BYTES + 4 * B bytes, zeroed once)
int ce_geom(const uint64_t* a, LaunchGeom* g) {
  g->grid = dim3((unsigned)a[4]); g->block = dim3(EW_THREADS); g->smem = 0; g->func = (const void*)ce_kernel;
  return 0;
}
int ce_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  ce_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (const int*)a[1], (float*)a[2], (float*)a[3], (int)a[4], (int)a[5],
                                       (unsigned char*)a[6], sig);
  CHECK_LAUNCH();
}

// ---- maxpool: args x, y, N, H, W, C, P, Q
int maxpool_geom(const uint64_t* a, LaunchGeom* g) {
  if (a[5] % 4 || (a[0] & 15) || (a[1] & 15)) return ORION_E_INVAL;   // channel quads, 128-bit aligned
  ew_geom(g, a[2] * a[6] * a[7] * (a[5] / 4), (const void*)maxpool_kernel);
  return 0;
}
int maxpool_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  maxpool_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (int)a[2], (int)a[3], (int)a[4], (int)a[5], (int)a[6],
                                            (int)a[7], sig);
  CHECK_LAUNCH();
}

// ---- avgpool: args x, y, N, HW, C ; bwd: dy, dx, N, HW, C
int avgpool_geom(const uint64_t* a, LaunchGeom* g) { ew_geom(g, a[2] * a[4], (const void*)avgpool_kernel); return 0; }
int avgpool_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  avgpool_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (int)a[2], (int)a[3], (int)a[4], sig);
  CHECK_LAUNCH();
}
int avgpool_bwd_geom(const uint64_t* a, LaunchGeom* g) { ew_geom(g, a[2] * a[3] * a[4], (const void*)avgpool_bwd_kernel); return 0; }
int avgpool_bwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  avgpool_bwd_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (int)a[2], (int)a[3], (int)a[4], sig);
  CHECK_LAUNCH();
}
