// Depthwise 3x3 convolution (groups = C; MobileNetV2's memory-bound conv), NHWC activations,
// weights [C][3][3][1]. fwd, stride-1 dgrad and wgrad slide a 3x3 register window along output
// rows (one warp = 32 channels x one row); stride-2 dgrad gathers per output pixel (4 channels per
// thread). wgrad reductions: fp32 per row, fp64 across rows, fixed-order CTA combine, ordered
// split reduction (combine_splits) per channel block.
#include "common.cuh"

namespace {

constexpr int DW_THREADS = 256;

struct DwShape { int N, H, W, C, stride, P, Q; };

// Row-blocked depthwise kernels: a warp owns 32 consecutive channels (128-byte coalesced rows of
// the NHWC tensor) and one output row (n, p); each lane produces U = 4 consecutive outputs per step
// from a 3 x ((U-1)*S+3) register window of its input columns whose loads are all issued
// together (memory-level parallelism instead of one dependent load per output). Weights live in
// registers. S = stride (compile-time 1 or 2).
constexpr int ROW_WARPS = 8;
constexpr int DW_U = 4;
constexpr int DW_UW = 8;   // wgrad: twice the loads in flight per window block (latency-bound, ncu r01)
constexpr int DW_U1 = 8;   // stride-1 fwd / dgrad: 8 outputs per 3 x 10 window (3.75 loads per output instead of 4.5)

template <int S, int U = DW_U>
struct Win {
  static constexpr int NC = (U - 1) * S + 3;   // input columns per block of U outputs
  float v[3][NC];
  // columns col0 .. col0+NC-1 of the 3 input rows (zero outside the image / missing rows)
  __device__ __forceinline__ void load(const float* const (&rowp)[3], const bool (&rv)[3], int col0, int W, int C) {
#pragma unroll
    for (int r = 0; r < 3; r++)
#pragma unroll
      for (int j = 0; j < NC; j++) {
        const int col = col0 + j;
        v[r][j] = (rv[r] && (unsigned)col < (unsigned)W) ? __ldg(rowp[r] + (long long)col * C) : 0.f;
      }
  }
};

template <int S>
__global__ void __launch_bounds__(DW_THREADS) dw_fwd_rows_kernel(const float* __restrict__ x, const float* __restrict__ w,
                                                                 float* __restrict__ y, DwShape s, OrionSig sig) {
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const int cblocks = (s.C + 31) / 32;
  const long long nrows = (long long)s.N * s.P;
  for (long long item = (long long)blockIdx.x * ROW_WARPS + warp; item < nrows * cblocks; item += (long long)gridDim.x * ROW_WARPS) {
    const int cb = (int)(item % cblocks);
    const long long row = item / cblocks;
    const int p = (int)(row % s.P), n = (int)(row / s.P);
    const int c = cb * 32 + lane;
    if (c >= s.C) continue;
    float wr[9];
#pragma unroll
    for (int t = 0; t < 9; t++) wr[t] = __ldg(w + c * 9 + t);
    const float* xr[3];
    bool rv[3];
#pragma unroll
    for (int r = 0; r < 3; r++) {
      int h = p * S - 1 + r;
      rv[r] = (unsigned)h < (unsigned)s.H;
      xr[r] = x + (((long long)n * s.H + (rv[r] ? h : 0)) * s.W) * s.C + c;
    }
    float* yr = y + (((long long)n * s.P + p) * s.Q) * s.C + c;
    constexpr int U = S == 1 ? DW_U1 : DW_U;
    for (int q0 = 0; q0 < s.Q; q0 += U) {
      Win<S, U> win;
      win.load(xr, rv, q0 * S - 1, s.W, s.C);
#pragma unroll
      for (int u = 0; u < U; u++) {
        if (q0 + u < s.Q) {
          float acc = 0.f;
#pragma unroll
          for (int r = 0; r < 3; r++)
#pragma unroll
            for (int t = 0; t < 3; t++) acc = fmaf(win.v[r][u * S + t], wr[r * 3 + t], acc);
          yr[(long long)(q0 + u) * s.C] = acc;
        }
      }
    }
  }
  orion_signal(sig);
}

// Stride-1 dgrad is a correlation with the flipped kernel: dx(h, w) = sum_{r,u} dy(h+1-r, w+1-u) k(r,u).
__global__ void __launch_bounds__(DW_THREADS) dw_dgrad_rows_s1_kernel(const float* __restrict__ dy, const float* __restrict__ w,
                                                                      float* __restrict__ dx, DwShape s, OrionSig sig) {
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const int cblocks = (s.C + 31) / 32;
  const long long nrows = (long long)s.N * s.H;
  for (long long item = (long long)blockIdx.x * ROW_WARPS + warp; item < nrows * cblocks; item += (long long)gridDim.x * ROW_WARPS) {
    const int cb = (int)(item % cblocks);
    const long long row = item / cblocks;
    const int h = (int)(row % s.H), n = (int)(row / s.H);
    const int c = cb * 32 + lane;
    if (c >= s.C) continue;
    float wr[9];
#pragma unroll
    for (int t = 0; t < 9; t++) wr[t] = __ldg(w + c * 9 + t);
    const float* gr[3];
    bool rv[3];
#pragma unroll
    for (int r = 0; r < 3; r++) {   // kernel row r reads dy row p = h + 1 - r
      int pp = h + 1 - r;
      rv[r] = (unsigned)pp < (unsigned)s.P;
      gr[r] = dy + (((long long)n * s.P + (rv[r] ? pp : 0)) * s.Q) * s.C + c;
    }
    float* dr = dx + (((long long)n * s.H + h) * s.W) * s.C + c;
    for (int w0 = 0; w0 < s.W; w0 += DW_U1) {
      Win<1, DW_U1> win;               // dy columns w0-1 .. w0+U
      win.load(gr, rv, w0 - 1, s.Q, s.C);
#pragma unroll
      for (int u = 0; u < DW_U1; u++) {
        if (w0 + u < s.W) {
          // column index in win for dy column (w0+u)+1-t is u + 2 - t
          float acc = 0.f;
#pragma unroll
          for (int r = 0; r < 3; r++)
#pragma unroll
            for (int t = 0; t < 3; t++) acc = fmaf(win.v[r][u + 2 - t], wr[r * 3 + t], acc);
          dr[(long long)(w0 + u) * s.C] = acc;
        }
      }
    }
  }
  orion_signal(sig);
}

// Stride-2 dgrad, row-blocked: for input row h only kernel rows r with (h+1-r) even contribute
// (one row for even h, two for odd h), and along w the pair (w = 2j, 2j+1) reads dy columns j and
// j+1 only: dx(2j) = sum_r dy(p_r, j) k(r,1); dx(2j+1) = sum_r dy(p_r, j+1) k(r,0) + dy(p_r, j) k(r,2).
__global__ void __launch_bounds__(DW_THREADS) dw_dgrad_rows_s2_kernel(const float* __restrict__ dy, const float* __restrict__ w,
                                                                      float* __restrict__ dx, DwShape s, OrionSig sig) {
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const int cblocks = (s.C + 31) / 32;
  const long long nrows = (long long)s.N * s.H;
  for (long long item = (long long)blockIdx.x * ROW_WARPS + warp; item < nrows * cblocks; item += (long long)gridDim.x * ROW_WARPS) {
    const int cb = (int)(item % cblocks);
    const long long row = item / cblocks;
    const int h = (int)(row % s.H), n = (int)(row / s.H);
    const int c = cb * 32 + lane;
    if (c >= s.C) continue;
    // up to two contributing kernel rows
    int rr[2], pp[2], nr = 0;
#pragma unroll
    for (int r = 0; r < 3; r++) {
      const int ph = h + 1 - r;
      if (ph >= 0 && (ph & 1) == 0 && ph / 2 < s.P) { rr[nr] = r; pp[nr] = ph / 2; nr++; }
    }
    float k0[2], k1[2], k2[2];
    const float* gr[2];
#pragma unroll
    for (int i = 0; i < 2; i++) {
      const bool on = i < nr;
      k0[i] = on ? __ldg(w + c * 9 + rr[i] * 3 + 0) : 0.f;
      k1[i] = on ? __ldg(w + c * 9 + rr[i] * 3 + 1) : 0.f;
      k2[i] = on ? __ldg(w + c * 9 + rr[i] * 3 + 2) : 0.f;
      gr[i] = dy + (((long long)n * s.P + (on ? pp[i] : 0)) * s.Q) * s.C + c;
    }
    auto ld = [&](int i, int col) -> float {
      return (i < nr && (unsigned)col < (unsigned)s.Q) ? __ldg(gr[i] + (long long)col * s.C) : 0.f;
    };
    float* dr = dx + (((long long)n * s.H + h) * s.W) * s.C + c;
    const int npairs = (s.W + 1) / 2;
    for (int j0 = 0; j0 < npairs; j0 += DW_U) {
      float col[2][DW_U + 1];
#pragma unroll
      for (int i = 0; i < 2; i++)
#pragma unroll
        for (int u = 0; u <= DW_U; u++) col[i][u] = ld(i, j0 + u);
#pragma unroll
      for (int u = 0; u < DW_U; u++) {
        const int we = 2 * (j0 + u);
        if (we < s.W) {
          float e = 0.f, o = 0.f;
#pragma unroll
          for (int i = 0; i < 2; i++) {
            e = fmaf(col[i][u], k1[i], e);
            o = fmaf(col[i][u + 1], k0[i], o);
            o = fmaf(col[i][u], k2[i], o);
          }
          dr[(long long)we * s.C] = e;
          if (we + 1 < s.W) dr[(long long)(we + 1) * s.C] = o;
        }
      }
    }
  }
  orion_signal(sig);
}

// wgrad: a warp accumulates the 9 taps of its 32 channels over whole output rows (register window
// blocks as above), fp32 per row and fp64 across rows; warps combine in smem in fixed order, CTAs
// write per-split partials, the last CTA of the channel block sums them in split order.
template <int S>
__global__ void __launch_bounds__(DW_THREADS, S == 1 ? 3 : 2) dw_wgrad_rows_kernel(const float* __restrict__ x, const float* __restrict__ dy,
                                                                   float* __restrict__ dw, DwShape s, unsigned char* ws, OrionSig sig) {
  __shared__ double sh[ROW_WARPS][9][32];
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const int c = blockIdx.x * 32 + lane;
  const long long nrows = (long long)s.N * s.P;
  // the fp64 row sums live in this lane's own shared-memory slots (no registers; same order)
  double* acc = &sh[warp][0][lane];
#pragma unroll
  for (int t = 0; t < 9; t++) acc[t * 32] = 0.0;
  if (c < s.C) {
    for (long long row = (long long)blockIdx.y * ROW_WARPS + warp; row < nrows; row += (long long)gridDim.y * ROW_WARPS) {
      const int p = (int)(row % s.P), n = (int)(row / s.P);
      const float* xr[3];
      bool rv[3];
#pragma unroll
      for (int r = 0; r < 3; r++) {
        int h = p * S - 1 + r;
        rv[r] = (unsigned)h < (unsigned)s.H;
        xr[r] = x + (((long long)n * s.H + (rv[r] ? h : 0)) * s.W) * s.C + c;
      }
      const float* gr = dy + (((long long)n * s.P + p) * s.Q) * s.C + c;
      float f[9];
#pragma unroll
      for (int t = 0; t < 9; t++) f[t] = 0.f;
      for (int q0 = 0; q0 < s.Q; q0 += DW_UW) {
        Win<S, DW_UW> win;
        win.load(xr, rv, q0 * S - 1, s.W, s.C);
        float g[DW_UW];
#pragma unroll
        for (int u = 0; u < DW_UW; u++) g[u] = (q0 + u < s.Q) ? __ldg(gr + (long long)(q0 + u) * s.C) : 0.f;
#pragma unroll
        for (int u = 0; u < DW_UW; u++)
#pragma unroll
          for (int r = 0; r < 3; r++)
#pragma unroll
            for (int t = 0; t < 3; t++) f[r * 3 + t] = fmaf(g[u], win.v[r][u * S + t], f[r * 3 + t]);
      }
#pragma unroll
      for (int t = 0; t < 9; t++) acc[t * 32] += (double)f[t];
    }
  }
  __syncthreads();
  unsigned int* tickets = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  if (warp == 0 && c < s.C) {
    for (int t = 0; t < 9; t++) {
      double v = 0.0;
      for (int wv = 0; wv < ROW_WARPS; wv++) v += sh[wv][t][lane];
      part[((long long)blockIdx.y * s.C + c) * 9 + t] = v;
    }
  }
  __shared__ double out[9 * 32];
  const int rs = gridDim.y, c0 = blockIdx.x * 32;
  const int V = 9 * min(32, s.C - c0);
  if (combine_splits(tickets + blockIdx.x * (combine_rows(rs) + 1), part + 9LL * c0, part + 9LL * rs * s.C + 9LL * c0, 9LL * s.C, rs,
                     blockIdx.y, V, out, &sh[0][0][0])) {
    for (int v = threadIdx.x; v < V; v += blockDim.x) dw[9LL * c0 + v] = (float)out[v];
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

DwShape dw_shape(const uint64_t* a) {
  // args: x|dy, w|dy, y|dx|dw, N, H, W, C, K(=C), R(=3), S(=3), stride, pad(=1), P, Q, [ws, ws_bytes]
  DwShape s;
  s.N = (int)a[3]; s.H = (int)a[4]; s.W = (int)a[5]; s.C = (int)a[6]; s.stride = (int)a[10]; s.P = (int)a[12]; s.Q = (int)a[13];
  return s;
}
bool dw_ok(const uint64_t* a) { return (a[6] % 4) == 0 && a[7] == a[6] && a[8] == 3 && a[9] == 3 && a[11] == 1; }

void ew(LaunchGeom* g, uint64_t n, const void* f, std::atomic<int>& occ) {
  uint64_t ctas = cdiv(n ? n : 1, DW_THREADS);
  const uint64_t wave = 148ull * resident_ctas_per_sm(f, DW_THREADS, occ);
  if (ctas > wave) ctas = wave;
  g->grid = dim3((unsigned)ctas); g->block = dim3(DW_THREADS); g->smem = 0; g->func = f;
}

void rows_geom(LaunchGeom* g, long long items, const void* f) {
  long long ctas = cdiv(items, ROW_WARPS);
  if (ctas > 148 * 8) ctas = 148 * 8;
  if (ctas < 1) ctas = 1;
  g->grid = dim3((unsigned)ctas); g->block = dim3(DW_THREADS); g->smem = 0; g->func = f;
}

int wg_splits(const DwShape& s) {
  long long cblocks = (s.C + 31) / 32;
  long long rs = cdiv(148 * 8, cblocks);
  long long max_rs = cdiv((long long)s.N * s.P, ROW_WARPS);
  if (rs > max_rs) rs = max_rs;
  if (rs < 1) rs = 1;
  return (int)rs;
}

}  // namespace

extern "C" uint64_t orion_dw_wgrad_workspace_bytes(uint64_t N, uint64_t C, uint64_t P, uint64_t Q) {
  DwShape s{(int)N, 0, 0, (int)C, 1, (int)P, (int)Q};
  const int rs = wg_splits(s);
  return WS_TICKET_BYTES + (uint64_t)(rs + combine_rows(rs)) * C * 9 * 8;
}

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

int dw_fwd_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if (s.stride != 1 && s.stride != 2) return ORION_E_INVAL;
  rows_geom(g, (long long)s.N * s.P * ((s.C + 31) / 32), s.stride == 1 ? (const void*)dw_fwd_rows_kernel<1> : (const void*)dw_fwd_rows_kernel<2>);
  return 0;
}
int dw_fwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  if (g.func == (const void*)dw_fwd_rows_kernel<1>)
    dw_fwd_rows_kernel<1><<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  else
    dw_fwd_rows_kernel<2><<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  CHECK_LAUNCH();
}
std::atomic<int> dw_dgrad_occ{0};
int dw_dgrad_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if (s.stride == 1) rows_geom(g, (long long)s.N * s.H * ((s.C + 31) / 32), (const void*)dw_dgrad_rows_s1_kernel);
  else if (s.stride == 2) rows_geom(g, (long long)s.N * s.H * ((s.C + 31) / 32), (const void*)dw_dgrad_rows_s2_kernel);
  else ew(g, (uint64_t)s.N * s.H * s.W * (s.C / 4), (const void*)dw_dgrad_kernel, dw_dgrad_occ);
  return 0;
}
int dw_dgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  if (g.func == (const void*)dw_dgrad_rows_s1_kernel)
    dw_dgrad_rows_s1_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  else if (g.func == (const void*)dw_dgrad_rows_s2_kernel)
    dw_dgrad_rows_s2_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  else
    dw_dgrad_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a), sig);
  CHECK_LAUNCH();
}
// wgrad args: x, dy, dw, N, H, W, C, C, 3, 3, stride, 1, P, Q, ws, ws_bytes
int dw_wgrad_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if (a[14] == 0 || a[15] < orion_dw_wgrad_workspace_bytes(s.N, s.C, s.P, s.Q)) return ORION_E_INVAL;
  if (s.stride != 1 && s.stride != 2) return ORION_E_INVAL;
  g->grid = dim3((s.C + 31) / 32, wg_splits(s)); g->block = dim3(DW_THREADS); g->smem = 0;
  g->func = s.stride == 1 ? (const void*)dw_wgrad_rows_kernel<1> : (const void*)dw_wgrad_rows_kernel<2>;
  return 0;
}
int dw_wgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  if (g.func == (const void*)dw_wgrad_rows_kernel<1>)
    dw_wgrad_rows_kernel<1><<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a),
                                                        (unsigned char*)a[14], sig);
  else
    dw_wgrad_rows_kernel<2><<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], dw_shape(a),
                                                        (unsigned char*)a[14], sig);
  CHECK_LAUNCH();
}
