// Depthwise 3x3 convolution (groups = C; MobileNetV2's memory-bound conv), NHWC activations,
// weights [C][3][3][1]. fwd, stride-1 dgrad and wgrad slide a 3x3 register window along output
// rows (one warp = 32 channels x one row); stride-2 dgrad gathers per output pixel (4 channels per
// thread). wgrad reductions: fp32 per row, fp64 across rows, fixed-order CTA combine, ordered
// split reduction (combine_splits) per channel block.
#include <cstdlib>

#include "common.cuh"

namespace {

constexpr int DW_THREADS = 256;

struct DwShape { int N, H, W, C, stride, P, Q; };

// Channel-quad kernels (round 2). A thread owns one channel quad (4 channels: 128-bit NHWC loads and
// stores; C % 4 == 0) and a segment of U consecutive outputs of one output row. It issues all the
// loads of its (U-1)*S+3-column input window at once (memory-level parallelism inside the thread),
// then forms the U output quads from registers: per output quad (U = 4, stride 1) 4.5 128-bit loads,
// 36 FFMA, one 128-bit store. The CTA stages the weights once as [tap][quad] float4s in shared
// memory. Items are (quad, segment, row) with the quad fastest, so a warp's loads are contiguous runs
// of NHWC rows. (Round 1 gave each lane one channel and recomputed a 64-bit address and a bounds
// predicate per scalar load: ~85 instructions per output; ncu: issue-bound at 77 % of issue slots,
// 29 % of DRAM bandwidth.)
__device__ __forceinline__ float4 ld4(const float* p, bool ok) {
  return ok ? __ldg(reinterpret_cast<const float4*>(p)) : make_float4(0.f, 0.f, 0.f, 0.f);
}
__device__ __forceinline__ void fma4(float4& a, const float4& x, const float4& w) {
  a.x = fmaf(x.x, w.x, a.x); a.y = fmaf(x.y, w.y, a.y); a.z = fmaf(x.z, w.z, a.z); a.w = fmaf(x.w, w.w, a.w);
}
// weights [C][3][3] -> shared [tap][C/4] float4 (FLIP: taps reversed, t -> 8 - t)
template <bool FLIP>
__device__ __forceinline__ void stage_taps(const float* __restrict__ w, int C, float4* wsm) {
  const int C4 = C / 4;
  for (int i = threadIdx.x; i < 9 * C4; i += blockDim.x) {
    const int t = i / C4, q = i % C4, c = q * 4, tt = FLIP ? 8 - t : t;
    wsm[i] = make_float4(__ldg(w + (c + 0) * 9 + tt), __ldg(w + (c + 1) * 9 + tt), __ldg(w + (c + 2) * 9 + tt), __ldg(w + (c + 3) * 9 + tt));
  }
  __syncthreads();
}
inline int dwq_smem(int C) { return 9 * (C / 4) * 16; }

// y[n,p,q,c] = sum_{r,u} x[n, p*S-1+r, q*S-1+u, c] k[c,r,u]; with FLIP (and S = 1, x = dy) this is
// the stride-1 data gradient dx[n,h,w,c] = sum_{r,u} dy[n,h+1-r,w+1-u,c] k[c,r,u].
//
// Round 3: a thread walks DOWN a band of output rows (fixed channel quad and segment of U outputs)
// with a rolling register window of the three input rows the taps read, so each input row is loaded
// once per segment (one new row per output row at stride 1, two at stride 2) instead of once per
// output row that reads it: 1.5 instead of 4.5 128-bit loads per output at stride 1, U = 4.
// Output rows per band: 16 for tall stride-1 maps (measured: 1.5 loads per output, 75 -> 63 us on
// MobileNetV2's 112x112x32 layer); stride 2 reuses only one of three input rows per step, so it keeps
// one row per item (more independent loads in flight; measured as fast as the band walk or faster).
__host__ __device__ inline int dw_bh(int P, int S) {
  if (S != 1) return 1;
  return P >= 32 ? 16 : (P > 16 ? (P + 1) / 2 : P);
}
template <int S, bool FLIP, int U>
__global__ void __launch_bounds__(DW_THREADS, 2) dw_q4_fwd_kernel(const float* __restrict__ x, const float* __restrict__ w,
                                                               float* __restrict__ y, int N, int H, int W, int C, int P, int Q,
                                                               OrionSig sig) {
  extern __shared__ float4 dwq_w[];
  stage_taps<FLIP>(w, C, dwq_w);
  constexpr int NC = (U - 1) * S + 3;
  const int C4 = C / 4, nseg = (Q + U - 1) / U, BH = dw_bh(P, S), nband = (P + BH - 1) / BH;
  const long long items = (long long)N * nband * nseg * C4;
  for (long long it = (long long)blockIdx.x * blockDim.x + threadIdx.x; it < items; it += (long long)gridDim.x * blockDim.x) {
    const int quad = (int)(it % C4);
    long long t2 = it / C4;
    const int q0 = (int)(t2 % nseg) * U;
    t2 /= nseg;
    const int band = (int)(t2 % nband), n = (int)(t2 / nband);
    const int p0 = band * BH, p1 = min(P, p0 + BH);
    const int c = quad * 4, w0 = q0 * S - 1;
    const float* xn = x + (long long)n * H * W * C + c;
    float4 win[3][NC];
    auto load_row = [&](float4 (&dst)[NC], int h) {
      const bool rv = (unsigned)h < (unsigned)H;
      const float* xr = xn + (long long)(rv ? h : 0) * W * C;
#pragma unroll
      for (int j = 0; j < NC; j++) dst[j] = ld4(xr + (long long)(w0 + j) * C, rv && (unsigned)(w0 + j) < (unsigned)W);
    };
    if (S == 1) {
      load_row(win[0], p0 - 1);
      load_row(win[1], p0);
    } else {
      load_row(win[2], 2 * p0 - 1);
    }
#pragma unroll 1
    for (int p = p0; p < p1; p++) {
      if (S == 1) {
        load_row(win[2], p + 1);
      } else {
#pragma unroll
        for (int j = 0; j < NC; j++) win[0][j] = win[2][j];
        load_row(win[1], 2 * p);
        load_row(win[2], 2 * p + 1);
      }
      // tap rows outer (three taps live at a time), same per-output order r, t as before
      float4 acc[U];
#pragma unroll
      for (int u = 0; u < U; u++) acc[u] = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int r = 0; r < 3; r++) {
        float4 k[3];
#pragma unroll
        for (int t = 0; t < 3; t++) k[t] = dwq_w[(r * 3 + t) * C4 + quad];
#pragma unroll
        for (int u = 0; u < U; u++)
#pragma unroll
          for (int t = 0; t < 3; t++) fma4(acc[u], win[r][u * S + t], k[t]);
      }
      float* yr = y + (((long long)n * P + p) * Q + q0) * C + c;
#pragma unroll
      for (int u = 0; u < U; u++)
        if (q0 + u < Q) *reinterpret_cast<float4*>(yr + (long long)u * C) = acc[u];
      if (S == 1) {
#pragma unroll
        for (int j = 0; j < NC; j++) { win[0][j] = win[1][j]; win[1][j] = win[2][j]; }
      }
    }
  }
  orion_signal(sig);
}

// Stride-2 data gradient: input row h takes kernel rows r with (h+1-r) even (dy row (h+1-r)/2);
// along w the pair (2j, 2j+1) reads dy columns j and j+1:
//   dx(2j) = sum_r dy(p_r, j) k(r,1);  dx(2j+1) = sum_r dy(p_r, j+1) k(r,0) + dy(p_r, j) k(r,2).
// Thread = (channel quad, segment of U pairs, input row): U+1 dy columns of <= 2 rows loaded at once.
template <int U>
__global__ void __launch_bounds__(DW_THREADS) dw_q4_dgrad_s2_kernel(const float* __restrict__ dy, const float* __restrict__ w,
                                                                    float* __restrict__ dx, int N, int H, int W, int C, int P, int Q,
                                                                    OrionSig sig) {
  extern __shared__ float4 dwq_w[];
  stage_taps<false>(w, C, dwq_w);
  const int C4 = C / 4, npairs = (W + 1) / 2, nseg = (npairs + U - 1) / U;
  const long long items = (long long)N * H * nseg * C4;
  for (long long it = (long long)blockIdx.x * blockDim.x + threadIdx.x; it < items; it += (long long)gridDim.x * blockDim.x) {
    const int quad = (int)(it % C4);
    long long t2 = it / C4;
    const int j0 = (int)(t2 % nseg) * U;
    const long long row = t2 / nseg;
    const int h = (int)(row % H), n = (int)(row / H);
    const int c = quad * 4;
    // odd h: kernel rows 0 and 2 (dy rows (h+1)/2 and (h-1)/2); even h: kernel row 1 (dy row h/2)
    const bool odd = h & 1;
    const int rsel[2] = {odd ? 0 : 1, 2};
    const int prow[2] = {odd ? (h + 1) / 2 : h / 2, (h - 1) / 2};
    const bool on[2] = {prow[0] < P, odd && prow[1] >= 0 && prow[1] < P};
    float4 g[2][U + 1];
#pragma unroll
    for (int i = 0; i < 2; i++) {
      const float* gr = dy + (((long long)n * P + (on[i] ? prow[i] : 0)) * Q) * C + c;
#pragma unroll
      for (int j = 0; j <= U; j++) g[i][j] = ld4(gr + (long long)(j0 + j) * C, on[i] && j0 + j < Q);
    }
    float4 k0[2], k1[2], k2[2];
#pragma unroll
    for (int i = 0; i < 2; i++) {
      k0[i] = dwq_w[(rsel[i] * 3 + 0) * C4 + quad];
      k1[i] = dwq_w[(rsel[i] * 3 + 1) * C4 + quad];
      k2[i] = dwq_w[(rsel[i] * 3 + 2) * C4 + quad];
    }
    float* dr = dx + (((long long)n * H + h) * W) * C + c;
#pragma unroll
    for (int u = 0; u < U; u++) {
      const int we = 2 * (j0 + u);
      if (we < W) {
        float4 e = make_float4(0.f, 0.f, 0.f, 0.f), o = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int i = 0; i < 2; i++) { fma4(e, g[i][u], k1[i]); fma4(o, g[i][u + 1], k0[i]); fma4(o, g[i][u], k2[i]); }
        *reinterpret_cast<float4*>(dr + (long long)we * C) = e;
        if (we + 1 < W) *reinterpret_cast<float4*>(dr + (long long)(we + 1) * C) = o;
      }
    }
  }
  orion_signal(sig);
}

// wgrad: dW[c,r,u] = sum_{n,p,q} dy[n,p,q,c] x[n, p*S-1+r, q*S-1+u, c]. A thread owns one channel
// quad and a segment of WU_ output columns of one image and walks DOWN a band of BH output rows
// with a rolling register window of the three x rows the taps read: per output row it loads only
// the new x rows (one for stride 1, two for stride 2) and the dy quads, so every x row is read once
// per segment (the round-2 row walker re-read each x row for three output rows and kept one
// segment's loads in flight per thread). The 36 tap sums accumulate in fp32 over the band (packed
// FFMA2), the CTA's lanes are summed in lane order in fp64, CTAs write per-split partials and the
// last CTA of the channel block sums them in split order (combine_splits): deterministic.
constexpr int WG_U = 2, WG_MAXQ = 64;

// output rows per band of the weight-gradient walker (measured A/B in one process, MobileNetV2 b96):
// 16 for the 112-row maps (103 us vs 107 / 118 at 32 / 64), 32 at stride 1 and the whole map at
// stride 2 for the 56-row ones (123 vs 141 us; 102 vs 127 us); the whole map below 32 rows
__host__ __device__ inline int wg_bh(int P, int S) {
  if (P >= 100) return 16;
  if (P >= 32) return S == 1 ? 32 : P;
  return P;
}

// lanes enumerate (segment, band, image), segment fastest; a CTA covers 256 / cq consecutive lanes
struct WgPlan { int cq, lanes, cblocks, nseg, nband, bh, rs; };
inline WgPlan wg_plan(int N, int C, int P, int Q, int S) {
  WgPlan w;
  const int C4 = C / 4;
  w.cq = C4 < WG_MAXQ ? C4 : WG_MAXQ;
  w.lanes = DW_THREADS / w.cq;
  w.cblocks = (int)cdiv(C4, w.cq);
  w.nseg = (int)cdiv(Q, WG_U);
  w.bh = wg_bh(P, S);
  w.nband = (int)cdiv(P, w.bh);
  w.rs = (int)cdiv((long long)N * w.nband * w.nseg, w.lanes);
  return w;
}

template <int S>
__global__ void __launch_bounds__(DW_THREADS, 2) dw_wgrad_band_kernel(const float* __restrict__ x, const float* __restrict__ dy,
                                                                      float* __restrict__ dwt, int N, int H, int W, int C, int P, int Q,
                                                                      int cq_n, int nseg, int nband, int BH, unsigned char* ws, OrionSig sig) {
  constexpr int NC = (WG_U - 1) * S + 3;   // x window columns of a segment
  extern __shared__ float wb_sh[];         // [lane][36][cq_n] fp32 band sums, later the fp64 combine area
  const int lanes = DW_THREADS / cq_n;
  const int cq = threadIdx.x % cq_n, lane = threadIdx.x / cq_n;
  const int c = (blockIdx.x * cq_n + cq) * 4;
  const long long Lg = (long long)blockIdx.y * lanes + lane;   // (segment fastest, band, image)
  const int seg = (int)(Lg % nseg);
  const long long t1 = Lg / nseg;
  const int band = (int)(t1 % nband), n = (int)(t1 / nband);
  float2 f[9][2];   // tap t: channels (c, c+1) and (c+2, c+3)
#pragma unroll
  for (int t = 0; t < 9; t++) { f[t][0] = make_float2(0.f, 0.f); f[t][1] = make_float2(0.f, 0.f); }
  if (lane < lanes && c < C && n < N) {
    const int p0 = band * BH, p1 = min(P, p0 + BH), q0 = seg * WG_U, w0 = q0 * S - 1;
    const float* xn = x + (long long)n * H * W * C + c;
    const float* gn = dy + (long long)n * P * Q * C + c;
    float4 win[3][NC];
    auto load_row = [&](float4 (&dst)[NC], int h) {
      const bool okh = (unsigned)h < (unsigned)H;
      const float* xr = xn + (long long)(okh ? h : 0) * W * C;
#pragma unroll
      for (int j = 0; j < NC; j++) dst[j] = ld4(xr + (long long)(w0 + j) * C, okh && (unsigned)(w0 + j) < (unsigned)W);
    };
    // rows p*S-1, p*S, p*S+1 of output row p: window rows 0..2
    if (S == 1) {
      load_row(win[0], p0 - 1);
      load_row(win[1], p0);
    } else {
      load_row(win[2], 2 * p0 - 1);
    }
#pragma unroll 1
    for (int p = p0; p < p1; p++) {
      if (S == 1) {
        load_row(win[2], p + 1);
      } else {
#pragma unroll
        for (int j = 0; j < NC; j++) win[0][j] = win[2][j];
        load_row(win[1], 2 * p);
        load_row(win[2], 2 * p + 1);
      }
      float4 g[WG_U];
      const float* gr = gn + (long long)p * Q * C;
#pragma unroll
      for (int u = 0; u < WG_U; u++) g[u] = ld4(gr + (long long)(q0 + u) * C, q0 + u < Q);
#pragma unroll
      for (int u = 0; u < WG_U; u++)
#pragma unroll
        for (int r = 0; r < 3; r++)
#pragma unroll
          for (int t = 0; t < 3; t++) {
            const float4 v = win[r][u * S + t];
            ffma2v(f[r * 3 + t][0], make_float2(g[u].x, g[u].y), make_float2(v.x, v.y));
            ffma2v(f[r * 3 + t][1], make_float2(g[u].z, g[u].w), make_float2(v.z, v.w));
          }
      if (S == 1) {
#pragma unroll
        for (int j = 0; j < NC; j++) { win[0][j] = win[1][j]; win[1][j] = win[2][j]; }
      }
    }
  }
  // lane sums: [lane][v][cq] fp32, v = tap*4 + channel-in-quad
  if (lane < lanes) {
#pragma unroll
    for (int t = 0; t < 9; t++) {
      float* d = wb_sh + ((size_t)lane * 36 + t * 4) * cq_n + cq;
      d[0] = f[t][0].x; d[(size_t)cq_n] = f[t][0].y; d[2 * (size_t)cq_n] = f[t][1].x; d[3 * (size_t)cq_n] = f[t][1].y;
    }
  }
  __syncthreads();
  unsigned int* tickets = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  const int c0 = blockIdx.x * cq_n * 4;
  const int nch = min(cq_n * 4, C - c0);
  // partial of this split: part[split][c][tap] (tap = r*3+u), lanes summed in lane order (fp64)
  for (int v = threadIdx.x; v < nch * 9; v += DW_THREADS) {
    const int cc = v / 9, t = v % 9, q4 = cc / 4, j = cc % 4;
    double sum = 0.0;
    for (int l = 0; l < lanes; l++) sum += (double)wb_sh[((size_t)l * 36 + t * 4 + j) * cq_n + q4];
    part[((long long)blockIdx.y * C + c0 + cc) * 9 + t] = sum;
  }
  const int rs = gridDim.y;
  const int V = 9 * nch;
  __syncthreads();
  double* out = reinterpret_cast<double*>(wb_sh);   // reuse (the partials above are in global memory now)
  if (combine_splits(tickets + blockIdx.x * (combine_rows(rs) + 1), part + 9LL * c0, part + 9LL * rs * C + 9LL * c0, 9LL * C, rs,
                     blockIdx.y, V, out, out + V)) {
    for (int v = threadIdx.x; v < V; v += DW_THREADS) dwt[9LL * c0 + v] = (float)out[v];
  }
  orion_signal(sig);
}
inline int wg_smem(const WgPlan& w) {
  const int lanesum = DW_THREADS * 36 * 4;                    // fp32 [lane][36][cq]
  const int comb = (9 * 4 * w.cq + DW_THREADS) * 8;           // fp64 combine area + scratch
  return lanesum > comb ? lanesum : comb;
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
bool dw_ok(const uint64_t* a) { return (a[6] % 4) == 0 && a[6] <= 2048 && a[7] == a[6] && a[8] == 3 && a[9] == 3 && a[11] == 1; }

void ew(LaunchGeom* g, uint64_t n, const void* f, std::atomic<int>& occ) {
  uint64_t ctas = cdiv(n ? n : 1, DW_THREADS);
  const uint64_t wave = 148ull * resident_ctas_per_sm(f, DW_THREADS, occ);
  if (ctas > wave) ctas = wave;
  g->grid = dim3((unsigned)ctas); g->block = dim3(DW_THREADS); g->smem = 0; g->func = f;
}

constexpr int DWQ_U1 = 4, DWQ_U2 = 2, DWQ_UP = 4;   // outputs (pairs) per thread item: stride 1 / stride 2 / s2 dgrad
std::atomic<int> dwq_occ[4];
// shared memory for the staged weights of up to C = 2048 channels (set once per kernel)
bool dwq_prepare() {
  static std::atomic<int> done{0};
  if (done.load(std::memory_order_acquire)) return true;
  const void* fs[4] = {(const void*)dw_q4_fwd_kernel<1, false, DWQ_U1>, (const void*)dw_q4_fwd_kernel<2, false, DWQ_U2>,
                       (const void*)dw_q4_fwd_kernel<1, true, DWQ_U1>, (const void*)dw_q4_dgrad_s2_kernel<DWQ_UP>};
  for (const void* f : fs)
    if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, dwq_smem(2048)) != cudaSuccess) {
      (void)cudaGetLastError();
      return false;
    }
  done.store(1, std::memory_order_release);
  return true;
}
void q4_geom(LaunchGeom* g, long long items, const void* f, std::atomic<int>& occ, int smem) {
  long long ctas = cdiv(items, DW_THREADS);
  int b = occ.load(std::memory_order_relaxed);   // resident CTAs per SM (occupancy query with this smem)
  if (b <= 0) {
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, f, DW_THREADS, smem) != cudaSuccess || b < 1) { (void)cudaGetLastError(); b = 4; }
    occ.store(b, std::memory_order_relaxed);
  }
  const long long wave = 148LL * b;   // one resident wave (shape heuristic, not the partition's count)
  if (ctas > wave) ctas = wave;
  if (ctas < 1) ctas = 1;
  g->grid = dim3((unsigned)ctas); g->block = dim3(DW_THREADS); g->smem = smem; g->func = f;
}

}  // namespace

extern "C" uint64_t orion_dw_wgrad_workspace_bytes(uint64_t N, uint64_t C, uint64_t P, uint64_t Q) {
  if (C % 4) C += 4 - C % 4;
  // (the stride is not an argument: size for the larger of the two plans)
  const WgPlan w1 = wg_plan((int)N, (int)C, (int)P, (int)Q, 1), w2 = wg_plan((int)N, (int)C, (int)P, (int)Q, 2);
  const int rs = w1.rs > w2.rs ? w1.rs : w2.rs;
  return WS_TICKET_BYTES + (uint64_t)(rs + combine_rows(rs)) * C * 9 * 8;
}

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

int dw_fwd_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if (s.stride != 1 && s.stride != 2) return ORION_E_INVAL;
  if (!dwq_prepare()) return ORION_E_CUDA;
  const int U = s.stride == 1 ? DWQ_U1 : DWQ_U2;
  const long long items = (long long)s.N * cdiv(s.P, dw_bh(s.P, s.stride)) * (s.C / 4) * cdiv(s.Q, U);
  if (s.stride == 1) q4_geom(g, items, (const void*)dw_q4_fwd_kernel<1, false, DWQ_U1>, dwq_occ[0], dwq_smem(s.C));
  else q4_geom(g, items, (const void*)dw_q4_fwd_kernel<2, false, DWQ_U2>, dwq_occ[1], dwq_smem(s.C));
  return 0;
}
int dw_fwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  DwShape s = dw_shape(a);
  if (g.func == (const void*)dw_q4_fwd_kernel<1, false, DWQ_U1>)
    dw_q4_fwd_kernel<1, false, DWQ_U1><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s.N, s.H, s.W, s.C,
                                                                       s.P, s.Q, sig);
  else
    dw_q4_fwd_kernel<2, false, DWQ_U2><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s.N, s.H, s.W, s.C,
                                                                       s.P, s.Q, sig);
  CHECK_LAUNCH();
}
std::atomic<int> dw_dgrad_occ{0};
int dw_dgrad_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if ((s.stride == 1 || s.stride == 2) && !dwq_prepare()) return ORION_E_CUDA;
  if (s.stride == 1)
    q4_geom(g, (long long)s.N * cdiv(s.H, dw_bh(s.H, 1)) * (s.C / 4) * cdiv(s.W, DWQ_U1),
            (const void*)dw_q4_fwd_kernel<1, true, DWQ_U1>, dwq_occ[2], dwq_smem(s.C));
  else if (s.stride == 2)
    q4_geom(g, (long long)s.N * s.H * (s.C / 4) * cdiv((s.W + 1) / 2, DWQ_UP), (const void*)dw_q4_dgrad_s2_kernel<DWQ_UP>, dwq_occ[3],
            dwq_smem(s.C));
  else ew(g, (uint64_t)s.N * s.H * s.W * (s.C / 4), (const void*)dw_dgrad_kernel, dw_dgrad_occ);
  return 0;
}
int dw_dgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  DwShape s = dw_shape(a);
  if (g.func == (const void*)dw_q4_fwd_kernel<1, true, DWQ_U1>)   // stride-1 dgrad = correlation of dy with the flipped kernel
    dw_q4_fwd_kernel<1, true, DWQ_U1><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s.N, s.P, s.Q, s.C,
                                                                      s.H, s.W, sig);
  else if (g.func == (const void*)dw_q4_dgrad_s2_kernel<DWQ_UP>)
    dw_q4_dgrad_s2_kernel<DWQ_UP><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s.N, s.H, s.W, s.C, s.P,
                                                                  s.Q, sig);
  else
    dw_dgrad_kernel<<<g.grid, g.block, 0, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s, sig);
  CHECK_LAUNCH();
}
// wgrad args: x, dy, dw, N, H, W, C, C, 3, 3, stride, 1, P, Q, ws, ws_bytes
int dw_wgrad_geom(const uint64_t* a, LaunchGeom* g) {
  if (!dw_ok(a)) return ORION_E_INVAL;
  DwShape s = dw_shape(a);
  if (a[14] == 0 || a[15] < orion_dw_wgrad_workspace_bytes(s.N, s.C, s.P, s.Q)) return ORION_E_INVAL;
  if (s.stride != 1 && s.stride != 2) return ORION_E_INVAL;
  const WgPlan w = wg_plan(s.N, s.C, s.P, s.Q, s.stride);
  if ((uint64_t)w.cblocks * (combine_rows(w.rs) + 1) * 4 > WS_TICKET_BYTES || w.rs > 65535) return ORION_E_INVAL;
  static std::atomic<int> attr{0};
  if (!attr.load()) {
    if (cudaFuncSetAttribute((const void*)dw_wgrad_band_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024) != cudaSuccess ||
        cudaFuncSetAttribute((const void*)dw_wgrad_band_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024) != cudaSuccess) {
      (void)cudaGetLastError();
      return ORION_E_CUDA;
    }
    attr.store(1);
  }
  g->grid = dim3((unsigned)w.cblocks, (unsigned)w.rs); g->block = dim3(DW_THREADS); g->smem = wg_smem(w);
  g->func = s.stride == 1 ? (const void*)dw_wgrad_band_kernel<1> : (const void*)dw_wgrad_band_kernel<2>;
  return 0;
}
int dw_wgrad_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t st) {
  DwShape s = dw_shape(a);
  const WgPlan w = wg_plan(s.N, s.C, s.P, s.Q, s.stride);
  if (g.func == (const void*)dw_wgrad_band_kernel<1>)
    dw_wgrad_band_kernel<1><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s.N, s.H, s.W, s.C, s.P, s.Q,
                                                            w.cq, w.nseg, w.nband, w.bh, (unsigned char*)a[14], sig);
  else
    dw_wgrad_band_kernel<2><<<g.grid, g.block, g.smem, st>>>((const float*)a[0], (const float*)a[1], (float*)a[2], s.N, s.H, s.W, s.C, s.P, s.Q,
                                                            w.cq, w.nseg, w.nband, w.bh, (unsigned char*)a[14], sig);
  CHECK_LAUNCH();
}
