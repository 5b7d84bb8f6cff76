// fp32 Transformer-encoder training operators (BE of BASELINE config 4: torch.nn.TransformerEncoderLayer
// stack, post-LN, ReLU FFN, trained in fp32 as the paper's PyTorch eager jobs are, P:955-962;
// reading R32): LayerNorm forward (saving mean / rstd) and backward, scaled-dot-product attention
// forward, and its backward in two ops (dQ with the per-query softmax statistics, then dK / dV).
// The Linear layers are liborion's fp32 GEMM (3xTF32 on tcgen05).
//
// Attention at the config's shape (S = 192, d = 64 per head) is small and latency-bound: the
// kernels keep a head's K and V (or Q and dO) in shared memory, give each warp 16 queries (keys),
// and run the dot products on the FMA pipe with each lane owning 6 keys (2 of the 64 output
// columns); softmax statistics use fixed xor-shuffle trees. Every output is produced by one lane in
// a fixed order: deterministic and partition-independent.
#include <float.h>
#include <atomic>

#include "common.cuh"

namespace {

#define CHECK_LAUNCH() return cudaGetLastError() == cudaSuccess ? 0 : ORION_E_CUDA

inline bool al16(uint64_t p) { return (p & 15) == 0; }

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// =========================================================================== LayerNorm fp32
// Warp per row, C % 128 == 0, C <= 512 (d_model of the config): each lane holds C/32 values.
constexpr int LN_T = 256, LN_MAXV = 4;   // float4 per lane
__global__ void __launch_bounds__(LN_T) ln_fwd_kernel(const float* __restrict__ x, float* __restrict__ y, const float* __restrict__ gamma,
                                                     const float* __restrict__ beta, float* __restrict__ mean_o, float* __restrict__ rstd_o,
                                                     long long rows, int C, float eps, OrionSig sig) {
  const int lane = threadIdx.x % 32;
  const long long row = (long long)blockIdx.x * (LN_T / 32) + threadIdx.x / 32;
  if (row < rows) {
    const int nv = C / 128;
    const float4* xr = reinterpret_cast<const float4*>(x + row * C);
    float4 v[LN_MAXV];
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < LN_MAXV; i++)
      if (i < nv) { v[i] = __ldg(xr + lane + 32 * i); s += (v[i].x + v[i].y) + (v[i].z + v[i].w); }
    const float mean = warp_sum(s) / (float)C;
    float q = 0.f;
#pragma unroll
    for (int i = 0; i < LN_MAXV; i++)
      if (i < nv) {
        const float a = v[i].x - mean, b = v[i].y - mean, c = v[i].z - mean, d = v[i].w - mean;
        q += (a * a + b * b) + (c * c + d * d);
      }
    const float rstd = 1.f / sqrtf(warp_sum(q) / (float)C + eps);
    float4* yr = reinterpret_cast<float4*>(y + row * C);
#pragma unroll
    for (int i = 0; i < LN_MAXV; i++)
      if (i < nv) {
        const float4 g = __ldg(reinterpret_cast<const float4*>(gamma) + lane + 32 * i);
        const float4 b = __ldg(reinterpret_cast<const float4*>(beta) + lane + 32 * i);
        float4 o;
        o.x = (v[i].x - mean) * rstd * g.x + b.x; o.y = (v[i].y - mean) * rstd * g.y + b.y;
        o.z = (v[i].z - mean) * rstd * g.z + b.z; o.w = (v[i].w - mean) * rstd * g.w + b.w;
        yr[lane + 32 * i] = o;
      }
    if (lane == 0) { mean_o[row] = mean; rstd_o[row] = rstd; }
  }
  orion_signal(sig);
}

// Backward: warp per row for dx (row means of g = dy*gamma and g*xhat by xor trees); the column
// sums dgamma = sum dy*xhat and dbeta = sum dy accumulate in fp64 per lane over the CTA's fixed
// contiguous row range, warps combine in order in shared memory, CTA partials are summed in CTA
// order by the last CTA (combine_splits).
constexpr int LNB_ROWS = 64;   // rows per CTA (shape-independent constant)
__global__ void __launch_bounds__(LN_T) ln_bwd_kernel(const float* __restrict__ x, const float* __restrict__ dy, float* __restrict__ dx,
                                                     const float* __restrict__ gamma, const float* __restrict__ mean_i,
                                                     const float* __restrict__ rstd_i, float* __restrict__ dgamma, float* __restrict__ dbeta,
                                                     long long rows, int C, unsigned char* ws, OrionSig sig) {
  extern __shared__ double lnb_sh[];   // [8 warps][2C] then scratch [LN_T]
  const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const int nv = C / 128;
  double pg[LN_MAXV][4], pb[LN_MAXV][4];
#pragma unroll
  for (int i = 0; i < LN_MAXV; i++)
#pragma unroll
    for (int e = 0; e < 4; e++) pg[i][e] = pb[i][e] = 0.0;
  const long long r0 = (long long)blockIdx.x * LNB_ROWS;
  const long long r1 = r0 + LNB_ROWS < rows ? r0 + LNB_ROWS : rows;
  for (long long row = r0 + warp; row < r1; row += LN_T / 32) {
    const float m = __ldg(mean_i + row), rs = __ldg(rstd_i + row);
    const float4* xr = reinterpret_cast<const float4*>(x + row * C);
    const float4* gr = reinterpret_cast<const float4*>(dy + row * C);
    float xh[LN_MAXV][4], gg[LN_MAXV][4];
    float s1 = 0.f, s2 = 0.f;
#pragma unroll
    for (int i = 0; i < LN_MAXV; i++)
      if (i < nv) {
        const float4 xv = __ldg(xr + lane + 32 * i), dv = __ldg(gr + lane + 32 * i);
        const float4 gm = __ldg(reinterpret_cast<const float4*>(gamma) + lane + 32 * i);
        const float xa[4] = {xv.x, xv.y, xv.z, xv.w}, da[4] = {dv.x, dv.y, dv.z, dv.w}, ga[4] = {gm.x, gm.y, gm.z, gm.w};
#pragma unroll
        for (int e = 0; e < 4; e++) {
          xh[i][e] = (xa[e] - m) * rs;
          gg[i][e] = da[e] * ga[e];
          s1 += gg[i][e];
          s2 += gg[i][e] * xh[i][e];
          pg[i][e] += (double)(da[e] * xh[i][e]);
          pb[i][e] += (double)da[e];
        }
      }
    const float mg = warp_sum(s1) / (float)C, mgx = warp_sum(s2) / (float)C;
    float4* dxr = reinterpret_cast<float4*>(dx + row * C);
#pragma unroll
    for (int i = 0; i < LN_MAXV; i++)
      if (i < nv) {
        float4 o;
        o.x = rs * (gg[i][0] - mg - xh[i][0] * mgx); o.y = rs * (gg[i][1] - mg - xh[i][1] * mgx);
        o.z = rs * (gg[i][2] - mg - xh[i][2] * mgx); o.w = rs * (gg[i][3] - mg - xh[i][3] * mgx);
        dxr[lane + 32 * i] = o;
      }
  }
  // warp partials -> shared (fixed layout), summed over warps in order
  double* wpart = lnb_sh;
#pragma unroll
  for (int i = 0; i < LN_MAXV; i++)
    if (i < nv)
#pragma unroll
      for (int e = 0; e < 4; e++) {
        const int c = (lane + 32 * i) * 4 + e;
        wpart[(long long)warp * 2 * C + c] = pg[i][e];
        wpart[(long long)warp * 2 * C + C + c] = pb[i][e];
      }
  __syncthreads();
  unsigned int* tk = reinterpret_cast<unsigned int*>(ws);
  double* part = reinterpret_cast<double*>(ws + WS_TICKET_BYTES);
  const int G = gridDim.x, V = 2 * C;
  for (int v = threadIdx.x; v < V; v += LN_T) {
    double s = 0.0;
    for (int w = 0; w < LN_T / 32; w++) s += wpart[(long long)w * V + v];
    part[(long long)blockIdx.x * V + v] = s;
  }
  double* gpart = part + (long long)G * V;
  double* out = gpart + (long long)combine_rows(G) * V;
  if (combine_splits(tk, part, gpart, V, G, blockIdx.x, V, out, lnb_sh + (LN_T / 32) * V)) {
    for (int v = threadIdx.x; v < C; v += LN_T) {
      dgamma[v] = (float)__ldcg(out + v);
      dbeta[v] = (float)__ldcg(out + C + v);
    }
  }
  orion_signal(sig);
}
inline int lnb_ctas(long long rows) { return (int)cdiv(rows, LNB_ROWS); }
inline uint64_t lnb_ws(long long rows, long long C) {
  const int G = lnb_ctas(rows);
  return WS_TICKET_BYTES + (uint64_t)(G + combine_rows(G) + 1) * 2 * C * 8;
}
inline int lnb_smem(int C) { return (LN_T / 32) * 2 * C * 8 + LN_T * 8; }

// ========================================================================== attention fp32
// Per (batch, head): D = 64 columns at h*64 of [B, S, ld] rows; S <= 256, S % 32 == 0.
constexpr int AD = 64, AQB = 64, AT = 256, AMAXK = 8;   // keys per lane: S / 32 <= 8
constexpr int AW = AT / 32;                             // warps per CTA (AQB / AW rows each)
constexpr int ACH = 4;                                  // independent partial sums per long reduction

// forward: O_i = sum_j softmax_j(q_i . k_j / sqrt d) v_j
__global__ void __launch_bounds__(AT) attn_fwd_kernel(const float* __restrict__ q, const float* __restrict__ k, const float* __restrict__ v,
                                                     float* __restrict__ o, int S, int ldi, int ldo, float scale, OrionSig sig) {
  extern __shared__ __align__(16) float asm_[];
  float* Ks = asm_;                       // [S][AD + 1]
  float* Vs = Ks + S * (AD + 1);          // [S][AD]
  float* Qs = Vs + S * AD;                // [4 warps][AD]
  float* Ps = Qs + AW * AD;               // [AW warps][S]
  const int b = blockIdx.z, h = blockIdx.y, lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const long long ib = (long long)b * S * ldi + h * AD, ob = (long long)b * S * ldo + h * AD;
  for (int e = threadIdx.x; e < S * AD / 4; e += AT) {
    const int r = e / (AD / 4), c = (e % (AD / 4)) * 4;
    const float4 kv = __ldg(reinterpret_cast<const float4*>(k + ib + (long long)r * ldi + c));
    Ks[r * (AD + 1) + c] = kv.x; Ks[r * (AD + 1) + c + 1] = kv.y; Ks[r * (AD + 1) + c + 2] = kv.z; Ks[r * (AD + 1) + c + 3] = kv.w;
    *reinterpret_cast<float4*>(Vs + r * AD + c) = __ldg(reinterpret_cast<const float4*>(v + ib + (long long)r * ldi + c));
  }
  __syncthreads();
  const int nk = S / 32;
  for (int qi = blockIdx.x * AQB + warp * (AQB / AW); qi < min(S, blockIdx.x * AQB + (warp + 1) * (AQB / AW)); qi++) {
    Qs[warp * AD + lane] = __ldg(q + ib + (long long)qi * ldi + lane);
    Qs[warp * AD + 32 + lane] = __ldg(q + ib + (long long)qi * ldi + 32 + lane);
    __syncwarp();
    float sc[AMAXK];
    float mx = -FLT_MAX;
#pragma unroll
    for (int t = 0; t < AMAXK; t++) {
      if (t < nk) {
        const float* kr = Ks + (lane + 32 * t) * (AD + 1);
        float a = 0.f;
#pragma unroll 16
        for (int c = 0; c < AD; c++) a = fmaf(Qs[warp * AD + c], kr[c], a);
        sc[t] = a * scale;
        mx = fmaxf(mx, sc[t]);
      }
    }
    mx = warp_max(mx);
    float l = 0.f;
#pragma unroll
    for (int t = 0; t < AMAXK; t++)
      if (t < nk) { sc[t] = expf(sc[t] - mx); l += sc[t]; Ps[warp * S + lane + 32 * t] = sc[t]; }
    l = warp_sum(l);
    __syncwarp();
    // ACH interleaved partial sums per output (the serial 192-term chain was latency-bound)
    float o0p[ACH], o1p[ACH];
#pragma unroll
    for (int i = 0; i < ACH; i++) { o0p[i] = 0.f; o1p[i] = 0.f; }
    for (int j = 0; j < S; j += ACH) {
#pragma unroll
      for (int i = 0; i < ACH; i++) {
        const float p = Ps[warp * S + j + i];
        o0p[i] = fmaf(p, Vs[(j + i) * AD + lane], o0p[i]);
        o1p[i] = fmaf(p, Vs[(j + i) * AD + 32 + lane], o1p[i]);
      }
    }
    const float o0 = (o0p[0] + o0p[1]) + (o0p[2] + o0p[3]), o1 = (o1p[0] + o1p[1]) + (o1p[2] + o1p[3]);
    const float rl = 1.f / l;
    o[ob + (long long)qi * ldo + lane] = o0 * rl;
    o[ob + (long long)qi * ldo + 32 + lane] = o1 * rl;
    __syncwarp();
  }
  orion_signal(sig);
}

// backward, op 1: per query i, P_ij recomputed, dP_ij = dO_i . v_j, Dl_i = sum_j P_ij dP_ij,
// dS_ij = P_ij (dP_ij - Dl_i), dQ_i = sum_j dS_ij k_j * scale. Also stores the row statistics
// (max m_i, 1/l_i, Dl_i) that op 2 needs to rebuild P and dS column-wise.
__global__ void __launch_bounds__(AT) attn_bwd_dq_kernel(const float* __restrict__ q, const float* __restrict__ k, const float* __restrict__ v,
                                                        const float* __restrict__ dO, float* __restrict__ dq, float* __restrict__ stats,
                                                        int S, int H, int ldi, int ldo, float scale, OrionSig sig) {
  extern __shared__ __align__(16) float asm_[];
  float* Ks = asm_;                       // [S][AD + 1]
  float* Vs = Ks + S * (AD + 1);          // [S][AD + 1]
  float* Qs = Vs + S * (AD + 1);          // [AW][AD]  (q row)
  float* Gs = Qs + AW * AD;               // [AW][AD]  (dO row)
  float* Ps = Gs + AW * AD;               // [AW][S]   (dS row)
  const int b = blockIdx.z, h = blockIdx.y, lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const long long ib = (long long)b * S * ldi + h * AD, ob = (long long)b * S * ldo + h * AD;
  for (int e = threadIdx.x; e < S * AD / 4; e += AT) {
    const int r = e / (AD / 4), c = (e % (AD / 4)) * 4;
    const float4 kv = __ldg(reinterpret_cast<const float4*>(k + ib + (long long)r * ldi + c));
    const float4 vv = __ldg(reinterpret_cast<const float4*>(v + ib + (long long)r * ldi + c));
    float* kd = Ks + r * (AD + 1) + c; float* vd = Vs + r * (AD + 1) + c;
    kd[0] = kv.x; kd[1] = kv.y; kd[2] = kv.z; kd[3] = kv.w;
    vd[0] = vv.x; vd[1] = vv.y; vd[2] = vv.z; vd[3] = vv.w;
  }
  __syncthreads();
  const int nk = S / 32;
  for (int qi = blockIdx.x * AQB + warp * (AQB / AW); qi < min(S, blockIdx.x * AQB + (warp + 1) * (AQB / AW)); qi++) {
    Qs[warp * AD + lane] = __ldg(q + ib + (long long)qi * ldi + lane);
    Qs[warp * AD + 32 + lane] = __ldg(q + ib + (long long)qi * ldi + 32 + lane);
    Gs[warp * AD + lane] = __ldg(dO + ob + (long long)qi * ldo + lane);
    Gs[warp * AD + 32 + lane] = __ldg(dO + ob + (long long)qi * ldo + 32 + lane);
    __syncwarp();
    float sc[AMAXK], dp[AMAXK];
    float mx = -FLT_MAX;
#pragma unroll
    for (int t = 0; t < AMAXK; t++) {
      if (t < nk) {
        const float* kr = Ks + (lane + 32 * t) * (AD + 1);
        const float* vr = Vs + (lane + 32 * t) * (AD + 1);
        float a = 0.f, g = 0.f;
#pragma unroll 16
        for (int c = 0; c < AD; c++) { a = fmaf(Qs[warp * AD + c], kr[c], a); g = fmaf(Gs[warp * AD + c], vr[c], g); }
        sc[t] = a * scale; dp[t] = g;
        mx = fmaxf(mx, sc[t]);
      }
    }
    mx = warp_max(mx);
    float l = 0.f;
#pragma unroll
    for (int t = 0; t < AMAXK; t++)
      if (t < nk) { sc[t] = expf(sc[t] - mx); l += sc[t]; }
    const float rl = 1.f / warp_sum(l);
    float dl = 0.f;
#pragma unroll
    for (int t = 0; t < AMAXK; t++)
      if (t < nk) { sc[t] *= rl; dl += sc[t] * dp[t]; }
    dl = warp_sum(dl);
#pragma unroll
    for (int t = 0; t < AMAXK; t++)
      if (t < nk) Ps[warp * S + lane + 32 * t] = sc[t] * (dp[t] - dl);
    __syncwarp();
    float g0p[ACH], g1p[ACH];
#pragma unroll
    for (int i = 0; i < ACH; i++) { g0p[i] = 0.f; g1p[i] = 0.f; }
    for (int j = 0; j < S; j += ACH) {
#pragma unroll
      for (int i = 0; i < ACH; i++) {
        const float ds = Ps[warp * S + j + i];
        g0p[i] = fmaf(ds, Ks[(j + i) * (AD + 1) + lane], g0p[i]);
        g1p[i] = fmaf(ds, Ks[(j + i) * (AD + 1) + 32 + lane], g1p[i]);
      }
    }
    const float g0 = (g0p[0] + g0p[1]) + (g0p[2] + g0p[3]), g1 = (g1p[0] + g1p[1]) + (g1p[2] + g1p[3]);
    dq[ib + (long long)qi * ldi + lane] = g0 * scale;
    dq[ib + (long long)qi * ldi + 32 + lane] = g1 * scale;
    if (lane == 0) {
      float* st = stats + (((long long)b * H + h) * S + qi) * 3;
      st[0] = mx; st[1] = rl; st[2] = dl;
    }
    __syncwarp();
  }
  orion_signal(sig);
}

// backward, op 2: per key j, P_ij = exp(s_ij - m_i) / l_i and dS_ij = P_ij (dO_i . v_j - Dl_i) from
// the stored row statistics; dV_j = sum_i P_ij dO_i, dK_j = sum_i dS_ij q_i * scale.
__global__ void __launch_bounds__(AT) attn_bwd_dkv_kernel(const float* __restrict__ q, const float* __restrict__ k, const float* __restrict__ v,
                                                         const float* __restrict__ dO, const float* __restrict__ stats, float* __restrict__ dk,
                                                         float* __restrict__ dv, int S, int H, int ldi, int ldo, float scale, OrionSig sig) {
  extern __shared__ __align__(16) float asm_[];
  float* Qs = asm_;                       // [S][AD + 1]
  float* Gs = Qs + S * (AD + 1);          // [S][AD + 1]  (dO)
  float* St = Gs + S * (AD + 1);          // [S][3]
  float* Ks = St + S * 3;                 // [AW][AD]
  float* Vw = Ks + AW * AD;               // [AW][AD]
  float* Pw = Vw + AW * AD;               // [AW][2][S]
  const int b = blockIdx.z, h = blockIdx.y, lane = threadIdx.x % 32, warp = threadIdx.x / 32;
  const long long ib = (long long)b * S * ldi + h * AD, ob = (long long)b * S * ldo + h * AD;
  for (int e = threadIdx.x; e < S * AD / 4; e += AT) {
    const int r = e / (AD / 4), c = (e % (AD / 4)) * 4;
    const float4 qv = __ldg(reinterpret_cast<const float4*>(q + ib + (long long)r * ldi + c));
    const float4 gv = __ldg(reinterpret_cast<const float4*>(dO + ob + (long long)r * ldo + c));
    float* qd = Qs + r * (AD + 1) + c; float* gd = Gs + r * (AD + 1) + c;
    qd[0] = qv.x; qd[1] = qv.y; qd[2] = qv.z; qd[3] = qv.w;
    gd[0] = gv.x; gd[1] = gv.y; gd[2] = gv.z; gd[3] = gv.w;
  }
  for (int e = threadIdx.x; e < S * 3; e += AT) St[e] = __ldg(stats + ((long long)b * H + h) * S * 3 + e);
  __syncthreads();
  const int nq = S / 32;
  for (int kj = blockIdx.x * AQB + warp * (AQB / AW); kj < min(S, blockIdx.x * AQB + (warp + 1) * (AQB / AW)); kj++) {
    Ks[warp * AD + lane] = __ldg(k + ib + (long long)kj * ldi + lane);
    Ks[warp * AD + 32 + lane] = __ldg(k + ib + (long long)kj * ldi + 32 + lane);
    Vw[warp * AD + lane] = __ldg(v + ib + (long long)kj * ldi + lane);
    Vw[warp * AD + 32 + lane] = __ldg(v + ib + (long long)kj * ldi + 32 + lane);
    __syncwarp();
#pragma unroll
    for (int t = 0; t < AMAXK; t++) {
      if (t < nq) {
        const int i = lane + 32 * t;
        const float* qr = Qs + i * (AD + 1);
        const float* gr = Gs + i * (AD + 1);
        float a = 0.f, g = 0.f;
#pragma unroll 16
        for (int c = 0; c < AD; c++) { a = fmaf(qr[c], Ks[warp * AD + c], a); g = fmaf(gr[c], Vw[warp * AD + c], g); }
        const float p = expf(a * scale - St[i * 3]) * St[i * 3 + 1];
        Pw[(warp * 2) * S + i] = p;
        Pw[(warp * 2 + 1) * S + i] = p * (g - St[i * 3 + 2]);
      }
    }
    __syncwarp();
    float v0p[ACH], v1p[ACH], k0p[ACH], k1p[ACH];
#pragma unroll
    for (int e = 0; e < ACH; e++) { v0p[e] = 0.f; v1p[e] = 0.f; k0p[e] = 0.f; k1p[e] = 0.f; }
    for (int i0 = 0; i0 < S; i0 += ACH) {
#pragma unroll
      for (int e = 0; e < ACH; e++) {
        const int i = i0 + e;
        const float p = Pw[(warp * 2) * S + i], ds = Pw[(warp * 2 + 1) * S + i];
        v0p[e] = fmaf(p, Gs[i * (AD + 1) + lane], v0p[e]);
        v1p[e] = fmaf(p, Gs[i * (AD + 1) + 32 + lane], v1p[e]);
        k0p[e] = fmaf(ds, Qs[i * (AD + 1) + lane], k0p[e]);
        k1p[e] = fmaf(ds, Qs[i * (AD + 1) + 32 + lane], k1p[e]);
      }
    }
    const float v0 = (v0p[0] + v0p[1]) + (v0p[2] + v0p[3]), v1 = (v1p[0] + v1p[1]) + (v1p[2] + v1p[3]);
    const float k0 = (k0p[0] + k0p[1]) + (k0p[2] + k0p[3]), k1 = (k1p[0] + k1p[1]) + (k1p[2] + k1p[3]);
    dv[ib + (long long)kj * ldi + lane] = v0;
    dv[ib + (long long)kj * ldi + 32 + lane] = v1;
    dk[ib + (long long)kj * ldi + lane] = k0 * scale;
    dk[ib + (long long)kj * ldi + 32 + lane] = k1 * scale;
    __syncwarp();
  }
  orion_signal(sig);
}
inline int attn_fwd_smem(int S) { return (S * (AD + 1) + S * AD + AW * AD + AW * S) * 4; }
inline int attn_dq_smem(int S) { return (2 * S * (AD + 1) + 2 * AW * AD + AW * S) * 4; }
inline int attn_dkv_smem(int S) { return (2 * S * (AD + 1) + 3 * S + 2 * AW * AD + 2 * AW * S) * 4; }
bool attn_prepare() {
  static std::atomic<int> done{0};
  if (done.load()) return true;
  const int mx = attn_dkv_smem(256) > attn_dq_smem(256) ? attn_dkv_smem(256) : attn_dq_smem(256);
  bool ok = cudaFuncSetAttribute((const void*)attn_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, attn_fwd_smem(256)) == cudaSuccess &&
            cudaFuncSetAttribute((const void*)attn_bwd_dq_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, mx) == cudaSuccess &&
            cudaFuncSetAttribute((const void*)attn_bwd_dkv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, mx) == cudaSuccess &&
            cudaFuncSetAttribute((const void*)ln_bwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, lnb_smem(128 * LN_MAXV)) == cudaSuccess;
  if (ok) done.store(1);
  return ok;
}

}  // namespace

extern "C" uint64_t orion_layernorm_bwd_workspace_bytes(uint64_t rows, uint64_t C) { return lnb_ws((long long)rows, (long long)C); }

// layernorm_f32: args x, y, gamma, beta, mean, rstd, rows, C, eps_bits
int layernorm_f32_geom(const uint64_t* a, LaunchGeom* g) {
  const long long rows = (long long)a[6], C = (long long)a[7];
  if (rows <= 0 || C <= 0 || C % 128 || C > 128 * LN_MAXV || !al16(a[0]) || !al16(a[1]) || !al16(a[2]) || !al16(a[3])) return ORION_E_INVAL;
  g->grid = dim3((unsigned)cdiv(rows, LN_T / 32)); g->block = dim3(LN_T); g->smem = 0; g->func = (const void*)ln_fwd_kernel;
  return 0;
}
int layernorm_f32_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  ln_fwd_kernel<<<g.grid, g.block, 0, s>>>((const float*)a[0], (float*)a[1], (const float*)a[2], (const float*)a[3], (float*)a[4], (float*)a[5],
                                           (long long)a[6], (int)a[7], u2f(a[8]), sig);
  CHECK_LAUNCH();
}
// layernorm_f32_bwd: args x, dy, dx, gamma, mean, rstd, dgamma, dbeta, rows, C, workspace, ws_bytes
int layernorm_f32_bwd_geom(const uint64_t* a, LaunchGeom* g) {
  const long long rows = (long long)a[8], C = (long long)a[9];
  if (rows <= 0 || C <= 0 || C % 128 || C > 128 * LN_MAXV || !al16(a[0]) || !al16(a[1]) || !al16(a[2]) || !al16(a[3])) return ORION_E_INVAL;
  if (a[10] == 0 || a[11] < lnb_ws(rows, C)) return ORION_E_INVAL;
  if (!attn_prepare()) return ORION_E_CUDA;
  g->grid = dim3((unsigned)lnb_ctas(rows)); g->block = dim3(LN_T); g->smem = lnb_smem((int)C); g->func = (const void*)ln_bwd_kernel;
  return 0;
}
int layernorm_f32_bwd_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  ln_bwd_kernel<<<g.grid, g.block, g.smem, s>>>((const float*)a[0], (const float*)a[1], (float*)a[2], (const float*)a[3], (const float*)a[4],
                                                (const float*)a[5], (float*)a[6], (float*)a[7], (long long)a[8], (int)a[9], (unsigned char*)a[10],
                                                sig);
  CHECK_LAUNCH();
}

// attention_f32: args q, k, v, o, B, S, heads, d, ld_in, ld_out
static int attn_check(const uint64_t* a, int np) {
  const long long B = (long long)a[np], S = (long long)a[np + 1], H = (long long)a[np + 2], d = (long long)a[np + 3];
  const long long ldi = (long long)a[np + 4], ldo = (long long)a[np + 5];
  if (B <= 0 || H <= 0 || d != AD || S <= 0 || S % 32 || S > 32 * AMAXK || ldi % 4 || ldo % 4 || ldi < H * d || ldo < H * d) return ORION_E_INVAL;
  for (int i = 0; i < np; i++)
    if (!al16(a[i])) return ORION_E_INVAL;
  return 0;
}
int attention_f32_geom(const uint64_t* a, LaunchGeom* g) {
  if (int r = attn_check(a, 4)) return r;
  if (!attn_prepare()) return ORION_E_CUDA;
  const int S = (int)a[5];
  g->grid = dim3((unsigned)cdiv(S, AQB), (unsigned)a[6], (unsigned)a[4]); g->block = dim3(AT); g->smem = attn_fwd_smem(S);
  g->func = (const void*)attn_fwd_kernel;
  return 0;
}
int attention_f32_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  attn_fwd_kernel<<<g.grid, g.block, g.smem, s>>>((const float*)a[0], (const float*)a[1], (const float*)a[2], (float*)a[3], (int)a[5],
                                                  (int)a[8], (int)a[9], 1.f / sqrtf((float)a[7]), sig);
  CHECK_LAUNCH();
}
// attention_f32_bwd_dq: args q, k, v, dO, dq, stats, B, S, heads, d, ld_in, ld_out
//   (q, k, v and dq rows of stride ld_in; dO of stride ld_out; stats [B][heads][S][3] fp32)
int attention_f32_bwd_dq_geom(const uint64_t* a, LaunchGeom* g) {
  if (int r = attn_check(a, 6)) return r;
  if (!attn_prepare()) return ORION_E_CUDA;
  const int S = (int)a[7];
  g->grid = dim3((unsigned)cdiv(S, AQB), (unsigned)a[8], (unsigned)a[6]); g->block = dim3(AT); g->smem = attn_dq_smem(S);
  g->func = (const void*)attn_bwd_dq_kernel;
  return 0;
}
int attention_f32_bwd_dq_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  attn_bwd_dq_kernel<<<g.grid, g.block, g.smem, s>>>((const float*)a[0], (const float*)a[1], (const float*)a[2], (const float*)a[3], (float*)a[4],
                                                     (float*)a[5], (int)a[7], (int)a[8], (int)a[10], (int)a[11], 1.f / sqrtf((float)a[9]), sig);
  CHECK_LAUNCH();
}
// attention_f32_bwd_dkv: args q, k, v, dO, stats, dk, dv, B, S, heads, d, ld_in, ld_out
int attention_f32_bwd_dkv_geom(const uint64_t* a, LaunchGeom* g) {
  if (int r = attn_check(a, 7)) return r;
  if (!attn_prepare()) return ORION_E_CUDA;
  const int S = (int)a[8];
  g->grid = dim3((unsigned)cdiv(S, AQB), (unsigned)a[9], (unsigned)a[7]); g->block = dim3(AT); g->smem = attn_dkv_smem(S);
  g->func = (const void*)attn_bwd_dkv_kernel;
  return 0;
}
int attention_f32_bwd_dkv_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s) {
  attn_bwd_dkv_kernel<<<g.grid, g.block, g.smem, s>>>((const float*)a[0], (const float*)a[1], (const float*)a[2], (const float*)a[3],
                                                      (const float*)a[4], (float*)a[5], (float*)a[6], (int)a[8], (int)a[9], (int)a[11], (int)a[12],
                                                      1.f / sqrtf((float)a[10]), sig);
  CHECK_LAUNCH();
}
