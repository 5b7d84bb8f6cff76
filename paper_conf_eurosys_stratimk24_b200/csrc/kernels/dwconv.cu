// Depthwise 3x3 convolution (groups = C; MobileNetV2's memory-bound conv, "MobileNet-v2"),
// NHWC activations, weights [C][3][3][1]. fwd / dgrad: one thread per 4 channels of an output
// pixel (128-bit loads along C). wgrad: per-thread fp64 accumulation of the 9 taps over a row
// split, fixed-order CTA combine, last CTA per channel block sums splits in order.
#include "common.cuh"

namespace {

constexpr int DW_THREADS = 256;

struct DwShape { int N, H, W, C, stride, P, Q; };

__global__ void __launch_bounds__(DW_THREADS) dw_fwd_kernel(const float* __restrict__ x, const float* __restrict__ w, float* __restrict__ y,
                                                            DwShape s, OrionSig sig) {
  const int C4 = s.C / 4;
  const long long total = (long long)s.N * s.P * s.Q * C4;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c4 = (int)(i % C4); long long t = i / C4;
    int q = (int)(t % s.Q); t /= s.Q;
    int p = (int)(t % s.P); int n = (int)(t / s.P);
    int c = c4 * 4;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int r = 0; r < 3; r++) {
      int h = p * s.stride - 1 + r;
      if ((unsigned)h >= (unsigned)s.H) continue;
#pragma unroll
      for (int u = 0; u < 3; u++) {
        int ww = q * s.stride - 1 + u;
        if ((unsigned)ww >= (unsigned)s.W) continue;
        float4 xv = __ldg(reinterpret_cast<const float4*>(x + (((long long)n * s.H + h) * s.W + ww) * s.C + c));
        int tap = r * 3 + u;
        acc.x = fmaf(xv.x, __ldg(w + (c + 0) * 9 + tap), acc.x);
        acc.y = fmaf(xv.y, __ldg(w + (c + 1) * 9 + tap), acc.y);
        acc.z = fmaf(xv.z, __ldg(w + (c + 2) * 9 + tap), acc.z);
        acc.w = fmaf(xv.w, __ldg(w + (c + 3) * 9 + tap), acc.w);
      }
    }
    reinterpret_cast<float4*>(y)[i] = acc;
  }
  orion_signal(sig);
}

// dx[n,h,w,c] = sum_{r,u} dy[n,p,q,c] * w[c,r,u] with h = p*stride - 1 + r
__global__ void __launch_bounds__(DW_THREADS) dw_dgrad_kernel(const float* __restrict__ dy, const float* __restrict__ w, float* __restrict__ dx,
                                                              DwShape s, OrionSig sig) {
  const int C4 = s.C / 4;
  const long long total = (long long)s.N * s.H * s.W * C4;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    int c4 = (int)(i % C4); long long t = i / C4;
    int wq = (int)(t % s.W); t /= s.W;
    int h = (int)(t % s.H); int n = (int)(t / s.H);
    int c = c4 * 4;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int r = 0; r < 3; r++) {
      int ph = h + 1 - r;
      if (ph < 0 || ph % s.stride) continue;
      int p = ph / s.stride;
      if (p >= s.P) continue;
#pragma unroll
      for (int u = 0; u < 3; u++) {
        int pw = wq + 1 - u;
        if (pw < 0 || pw % s.stride) continue;
        int q = pw / s.stride;
        if (q >= s.Q) continue;
        float4 g = __ldg(reinterpret_cast<const float4*>(dy + (((long long)n * s.P + p) * s.Q + q) * s.C + c));
        int tap = r * 3 + u;
        acc.x = fmaf(g.x, __ldg(w + (c + 0) * 9 + tap), acc.x);
        acc.y = fmaf(g.y, __ldg(w + (c + 1) * 9 + tap), acc.y);
        acc.z = fmaf(g.z, __ldg(w + (c + 2) * 9 + tap), acc.z);
        acc.w = fmaf(g.w, __ldg(w + (c + 3) * 9 + tap), acc.w);
      }
    }
    reinterpret_cast<float4*>(dx)[i] = acc;
  }
  orion_signal(sig);
}

// dw[c, r, u] = sum_{n,p,q} dy[n,p,q,c] x[n, p*st-1+r, q*st-1+u, c]
constexpr int WG_CB = 32;  // channels per CTA (one per lane), 8 position-lanes
__global__ void __launch_bounds__(DW_THREADS) dw_wgrad_kernel(const float* __restrict__ x, const float* __restrict__ dy, float* __restrict__ dw,
                                                              DwShape s, long long pos_per_split, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[DW_THREADS][9];
  const int cl = threadIdx.x % WG_CB, pl = threadIdx.x / WG_CB, PL = DW_THREADS / WG_CB;
  const int c = blockIdx.x * WG_CB + cl;
  const long long npos = (long long)s.N * s.P * s.Q;
  const long long p0 = blockIdx.y * pos_per_split, p1 = min(npos, p0 + pos_per_split);
  double acc[9];
#pragma unroll
  for (int j = 0; j < 9; j++) acc[j] = 0.0;
  if (c < s.C) {
    for (long long pos = p0 + pl; pos < p1; pos += PL) {
      int q = (int)(pos % s.Q); long long t = pos / s.Q;
      int p = (int)(t % s.P); int n = (int)(t / s.P);
      float g = __ldg(dy + pos * s.C + c);
#pragma unroll
      for (int r = 0; r < 3; r++) {
        int h = p * s.stride - 1 + r;
        if ((unsigned)h >= (unsigned)s.H) continue;
#pragma unroll
        for (int u = 0; u < 3; u++) {
          int ww = q * s.stride - 1 + u;
          if ((unsigned)ww >= (unsigned)s.W) continue;
          acc[r * 3 + u] += (double)g * (double)__ldg(x + (((long long)n * s.H + h) * s.W + ww) * s.C + c);
        }
      }
    }
  }
#pragma unroll
  for (int j = 0; j < 9; j++) sh[threadIdx.x][j] = acc[j];
  __syncthreads();
  unsigned int* tickets = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  if (pl == 0 && c < s.C) {
    for (int j = 0; j < 9; j++) {
      double t = 0.0;
      for (int r = 0; r < PL; r++) t += sh[r * WG_CB + cl][j];
      part[((long long)blockIdx.y * s.C + c) * 9 + j] = t;
    }
  }
  if (last_cta_of(tickets + blockIdx.x, gridDim.y)) {
    if (pl == 0 && c < s.C) {
      for (int j = 0; j < 9; j++) {
        double t = 0.0;
        for (unsigned r = 0; r < gridDim.y; r++) t += __ldcg(part + ((long long)r * s.C + c) * 9 + j);
        dw[c * 9 + j] = (float)t;
      }
    }
  }
  orion_signal(sig);
}

DwShape dw_shape(const uint64_t* a) {
  // args: x|dy, w|dy, y|dx|dw, N, H, W, C, K(=C), R(=3), S(=3), stride, pad(=1), P, Q, [ws, ws_bytes]
  DwShape s;
  s.N = (int)a[3]; s.H = (int)a[4]; s.W = (int)a[5]; s.C = (int)a[6]; s.stride = (int)a[10]; s.P = (int)a[12]; s.Q = (int)a[13];
  return s;
}
bool dw_ok(const uint64_t* a) { return (a[6] % 4) == 0 && a[7] == a[6] && a[8] == 3 && a[9] == 3 && a[11] == 1; }

void ew(LaunchGeom* g, uint64_t n, const void* f) {
  uint64_t ctas = cdiv(n ? n : 1, DW_THREADS);
  if (ctas > 148 * 8) ctas = 148 * 8;
  g->grid = dim3((unsigned)ctas); g->block = dim3(DW_THREADS); g->smem = 0; g->func = f;
}

struct WgSplit { int cblocks, rs; long long per; };
WgSplit wg_split(const DwShape& s) {
  WgSplit w;
  w.cblocks = (s.C + WG_CB - 1) / WG_CB;
  long long npos = (long long)s.N * s.P * s.Q;
  long long rs = cdiv(296, w.cblocks);
  long long max_rs = cdiv(npos, 256);
  if (rs > max_rs) rs = max_rs;
  if (rs < 1) rs = 1;
  w.rs = (int)rs;
  w.per = cdiv(npos, rs);
  return w;
}

}  // namespace

extern "C" uint64_t orion_dw_wgrad_workspace_bytes(uint64_t N, uint64_t C, uint64_t P, uint64_t Q) {
  DwShape s{(int)N, 0, 0, (int)C, 1, (int)P, (int)Q};
  WgSplit w = wg_split(s);
  return WS_TICKET_BYTES + (uint64_t)w.rs * C * 9 * 8;
}

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

int dw_fwd_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  ew(g, (uint64_t)s.N * s.P * s.Q * (s.C / 4), (const void*)dw_fwd_kernel);
  return 0;
}
int dw_fwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  dw_fwd_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  CHECK_LAUNCH();
}
int dw_dgrad_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  ew(g, (uint64_t)s.N * s.H * s.W * (s.C / 4), (const void*)dw_dgrad_kernel);
  return 0;
}
int dw_dgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  dw_dgrad_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  CHECK_LAUNCH();
}
// wgrad args: x, dy, dw, N, H, W, C, C, 3, 3, stride, 1, P, Q, ws, ws_bytes
int dw_wgrad_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if (a[14] == 0 || a[15] < orion_dw_wgrad_workspace_bytes(s.N, s.C, s.P, s.Q)) return ORION_E_INVAL;
  WgSplit w = wg_split(s);
  g->grid = dim3(w.cblocks, w.rs); g->block = dim3(DW_THREADS); g->smem = 0; g->func = (const void*)dw_wgrad_kernel;
  return 0;
}
int dw_wgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  DwShape s = dw_shape(a);
  WgSplit w = wg_split(s);
  dw_wgrad_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s, w.per, (unsigned char*)a[14], sig);
  CHECK_LAUNCH();
}
