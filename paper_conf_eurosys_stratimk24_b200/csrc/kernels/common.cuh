// Shared device/host plumbing of the operator kernels (not of the oracle).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "orion.h"
#include "orion_kernels.h"

#include <atomic>

// Resident CTAs per SM of a grid-stride kernel, from the occupancy query (cached per kernel in
// `slot`; 8 when the query fails, e.g. no device). The memory-bound grid-stride kernels cap their
// grid at one full wave of 148 SMs x this, so no CTA waits for a tail wave (results never depend
// on the grid size).
inline int resident_ctas_per_sm(const void* f, int threads, std::atomic<int>& slot) {
  int b = slot.load(std::memory_order_relaxed);
  if (b > 0) return b;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, f, threads, 0) != cudaSuccess || b < 1 || b > 8) {
    (void)cudaGetLastError();
    b = 8;
  }
  slot.store(b, std::memory_order_relaxed);
  return b;
}

// Completion signal fused into every kernel: the last CTA of a launch publishes `seq` (the
// client's completed-op count) to a host-mapped counter, so the scheduler observes completion by a
// plain load instead of a CUDA event query (P:778-786 uses cudaEventQuery).
struct OrionSig {
  unsigned long long* ticket;  // per-stream device counter of finished CTAs (monotone)
  unsigned long long* done;    // host-mapped completion counter of the stream
  unsigned long long target;   // ticket value reached when the last CTA of this launch finishes
  unsigned long long seq;      // value to publish
};

__device__ __forceinline__ void orion_signal(const OrionSig& sig) {
  if (sig.ticket == nullptr) return;  // direct launch (no scheduler)
  // Completion only: the counter tells the scheduler THAT the launch finished (HP busy test, BE
  // in-flight accounting); no consumer reads the kernel's data through it (later kernels and the
  // D2H memops see the data by stream order), so no memory fence is needed -- a gpu- and a
  // system-scope fence per kernel cost microseconds on the HP critical path (tools/diag_launch.py).
  // bar.sync: every thread of this CTA has finished before its CTA is counted.
  __syncthreads();
  if (threadIdx.x == 0 && threadIdx.y == 0 && threadIdx.z == 0) {
    unsigned long long t;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], 1;" : "=l"(t) : "l"(sig.ticket) : "memory");
    if (t + 1ull == sig.target) asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(sig.done), "l"(sig.seq) : "memory");
  }
}

// Launch geometry computed from the op's args (identical for geometry queries and launches).
struct LaunchGeom {
  dim3 grid{1, 1, 1}, block{1, 1, 1};
  int smem = 0;
  const void* func = nullptr;
  int pipe = 0;   // ORION_PIPE_*: the pipe the chosen kernel's arithmetic runs on (profiler ridge, R16)
  // CTAs that run orion_signal (0 = all of grid): an op that launches a second, signalling kernel
  // after an unsignalled one (split-K partials + their ordered combine) reports the second's grid
  unsigned long long sig_ctas = 0;
  unsigned long long signal_ctas() const { return sig_ctas ? sig_ctas : ctas(); }
  unsigned long long ctas() const { return (unsigned long long)grid.x * grid.y * grid.z; }
};

typedef int (*geom_fn)(const uint64_t* a, LaunchGeom* g);
typedef int (*launch_fn)(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);

struct KernelEntry {
  const char* name;
  int nargs;
  geom_fn geom;
  launch_fn launch;
};

__host__ __device__ __forceinline__ float u2f(uint64_t v) {
  union { uint32_t u; float f; } c; c.u = (uint32_t)v; return c.f;
}

__host__ __device__ __forceinline__ uint64_t cdiv(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// Packed fp32 FMA (sm_100a FFMA2): d.x += a * b.x, d.y += a * b.y, each lane rounded once exactly as
// fmaf would (same results bit for bit), one issue slot for two FMAs. The scalar a is broadcast to
// both lanes (SASS: FFMA2 Rd, Ra.F32, Rb.F32x2, Rd.F32x2).
__device__ __forceinline__ void ffma2(float2& d, float a, float2 b) {
  asm("{\n\t.reg .b64 a2, b2, d2;\n\tmov.b64 a2, {%2, %2};\n\tmov.b64 b2, {%3, %4};\n\tmov.b64 d2, {%0, %1};\n\t"
      "fma.rn.f32x2 d2, a2, b2, d2;\n\tmov.b64 {%0, %1}, d2;\n\t}"
      : "+f"(d.x), "+f"(d.y)
      : "f"(a), "f"(b.x), "f"(b.y));
}
// d.x += a.x * b.x, d.y += a.y * b.y (packed, each lane rounded once like fmaf)
__device__ __forceinline__ void ffma2v(float2& d, float2 a, float2 b) {
  asm("{\n\t.reg .b64 a2, b2, d2;\n\tmov.b64 a2, {%2, %3};\n\tmov.b64 b2, {%4, %5};\n\tmov.b64 d2, {%0, %1};\n\t"
      "fma.rn.f32x2 d2, a2, b2, d2;\n\tmov.b64 {%0, %1}, d2;\n\t}"
      : "+f"(d.x), "+f"(d.y)
      : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
}

// Last-CTA-of-a-group detection for deterministic two-phase reductions: every CTA of the group
// calls this after writing its partials; returns true in exactly one CTA (the last), which then
// reduces the partials in a fixed order. The ticket is reset by the last CTA.
__device__ __forceinline__ bool last_cta_of(unsigned int* ticket, unsigned int count) {
  __shared__ unsigned int s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();   // cumulative over the CTA's writes ordered before it by bar.sync
    unsigned int t = atomicAdd(ticket, 1u) + 1u;
    s_last = (t == count);
    if (t == count) *ticket = 0u;  // reset for the next launch (stream order serialises launches)
  }
  __syncthreads();
  if (s_last) __threadfence();
  return s_last != 0;
}

// Workspace layout shared by all ops of a client (they run in stream order): the first
// WS_TICKET_BYTES hold u32 tickets, always zero between launches (each group's last CTA resets its
// ticket); per-launch partials follow. Separating the two keeps one op's partials from ever
// aliasing another op's tickets.
constexpr uint64_t WS_TICKET_BYTES = 65536;

// dst[v] = sum_{z < n} src[z * stride + v] for v < V, summed in z order, by all threads of the
// CTA: value v gets T = blockDim / V threads (at least 1), thread j of them sums the fixed
// contiguous chunk j of the n rows (8 loads in flight), and the T chunk sums are added in chunk
// order. The split into chunks depends on (n, V, blockDim) only, so the result is deterministic.
// scratch: >= blockDim doubles of shared memory. dst may be global or shared; on return (after
// a barrier) dst is complete.
// (src may be fp32 or fp64 partials; the sums are fp64 either way)
template <class Src>
__device__ __forceinline__ double sum_chunk(const Src* src, long long stride, int z0, int z1, int v) {
  double s = 0.0;
  int z = z0;
  for (; z + 7 < z1; z += 8) {
    Src a[8];
#pragma unroll
    for (int i = 0; i < 8; i++) a[i] = __ldcg(src + (long long)(z + i) * stride + v);
#pragma unroll
    for (int i = 0; i < 8; i++) s += a[i];
  }
  for (; z < z1; z++) s += __ldcg(src + (long long)z * stride + v);
  return s;
}
// sum_rows_ordered: every value is summed over the rows in row order (unchanged results); a thread
// owns SR_VB consecutive values and keeps 8 rows x SR_VB loads in flight per batch, so a large V
// costs V / (SR_VB * blockDim) batches instead of V / blockDim dependent row walks.
constexpr int SR_VB = 4;
template <class Src>
__device__ inline void sum_rows_ordered(const Src* src, long long stride, int n, int V, double* dst, double* scratch) {
  const int nt = blockDim.x, t = threadIdx.x;
  if (V >= nt / 2) {
    for (int v0 = t * SR_VB; v0 < V; v0 += nt * SR_VB) {
      double acc[SR_VB];
#pragma unroll
      for (int j = 0; j < SR_VB; j++) acc[j] = 0.0;
      int z = 0;
      for (; z + 7 < n; z += 8) {
        Src a[8][SR_VB];
#pragma unroll
        for (int i = 0; i < 8; i++)
#pragma unroll
          for (int j = 0; j < SR_VB; j++) a[i][j] = v0 + j < V ? __ldcg(src + (long long)(z + i) * stride + v0 + j) : Src(0);
#pragma unroll
        for (int i = 0; i < 8; i++)
#pragma unroll
          for (int j = 0; j < SR_VB; j++) acc[j] += a[i][j];
      }
      for (; z < n; z++)
#pragma unroll
        for (int j = 0; j < SR_VB; j++)
          if (v0 + j < V) acc[j] += __ldcg(src + (long long)z * stride + v0 + j);
#pragma unroll
      for (int j = 0; j < SR_VB; j++)
        if (v0 + j < V) dst[v0 + j] = acc[j];
    }
  } else {
    int T = nt / V;
    if (T > n) T = n > 0 ? n : 1;
    const int v = t % V, j = t / V;
    if (j < T) scratch[j * V + v] = sum_chunk(src, stride, (int)((long long)j * n / T), (int)((long long)(j + 1) * n / T), v);
    __syncthreads();
    if (t < V) {
      double s = 0.0;
      for (int k = 0; k < T; k++) s += scratch[k * V + t];
      dst[t] = s;
    }
  }
  __syncthreads();
}

// Ordered combine of per-split partial vectors, two levels when there are many splits. Split z of
// a reduction (nz splits) has written its V values at part[z * stride ..]; the group partials
// live at gpart[g * stride ..] (ng = ceil(nz / G) rows). Tickets: tk[0] final, tk[1 + g] per
// group (zero at rest; reset by their last CTA). Level 1: the last CTA of each run of G
// consecutive splits sums the run in order into gpart[g]; level 2: the last run sums the gpart
// rows in order into out (shared, V doubles). Returns true in exactly one CTA, with out complete.
// G is a function of nz only (combine_group), so results do not depend on the SM partition.
__host__ __device__ __forceinline__ int combine_group(int nz) {
  if (nz <= 16) return nz;
  int g = 8;
  while (g * g < nz) g++;
  return g;
}
__host__ __device__ __forceinline__ int combine_rows(int nz) {   // gpart rows needed (0: one level)
  return nz <= 16 ? 0 : (nz + combine_group(nz) - 1) / combine_group(nz);
}
template <class Src>
__device__ inline bool combine_splits(unsigned int* tk, const Src* part, double* gpart, long long stride, int nz, int z, int V,
                                      double* out, double* scratch) {
  if (nz <= 16) {
    if (!last_cta_of(tk, (unsigned)nz)) return false;
    sum_rows_ordered(part, stride, nz, V, out, scratch);
    return true;
  }
  const int G = combine_group(nz), ng = (nz + G - 1) / G, g = z / G;
  const int gsize = min(G, nz - g * G);
  if (!last_cta_of(tk + 1 + g, (unsigned)gsize)) return false;
  sum_rows_ordered(part + (long long)g * G * stride, stride, gsize, V, gpart + (long long)g * stride, scratch);
  if (!last_cta_of(tk, (unsigned)ng)) return false;
  sum_rows_ordered(gpart, stride, ng, V, out, scratch);
  return true;
}

// Streaming weight-gradient GEMM (wgs.cu), taken by gemm flags = 1 when its TMA constraints hold.
uint64_t wgs_ws_bytes(long long M, long long N, long long K);
bool wgs_try_geom(const uint64_t* a, LaunchGeom* g);
bool wgs_is(const void* f);
int wgs_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);

// Tensor-core weight-gradient GEMM (atc.cu), taken by gemm flags = 1 for compute-dense shapes.
uint64_t atc_ws_bytes(long long M, long long N, long long K);
bool atc_try_geom(const uint64_t* a, LaunchGeom* g);
bool atc_is(const void* f);
int atc_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);
uint64_t atc_conv_ws_bytes(uint64_t N, uint64_t H, uint64_t W, uint64_t C, uint64_t K, uint64_t R, uint64_t S, uint64_t stride,
                           uint64_t pad);
bool atc_conv_try_geom(const uint64_t* a, LaunchGeom* g);
bool atc_conv_is(const void* f);
int atc_conv_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);

// Streaming tensor-core weight-gradient GEMM (ats.cu): long K, narrow operands, 3xTF32 on tcgen05.
uint64_t ats_ws_bytes(long long M, long long N, long long K);
bool ats_try_geom(const uint64_t* a, LaunchGeom* g);
bool ats_is(const void* f);
int ats_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);

// Forward convolution / dense B^T GEMM on tcgen05 with TMA im2col boxes (cvf.cu).
bool cvf_conv_try_geom(const uint64_t* a, LaunchGeom* g);
bool cvf_gemm_try_geom(const uint64_t* a, LaunchGeom* g);
bool cvf_is(const void* f);
int cvf_conv_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);
int cvf_gemm_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);

// Kernel table (table.cu)
extern const KernelEntry g_kernels[ORION_FN_COUNT];
int kernel_launch_sig(uint32_t fn, const uint64_t* args, uint32_t nargs, OrionSig sig, cudaStream_t s,
                      unsigned long long* ctas_out);

#define ENTRY_DECL(name) \
  int name##_geom(const uint64_t* a, LaunchGeom* g); \
  int name##_launch(const uint64_t* a, const LaunchGeom& g, OrionSig sig, cudaStream_t s);
ENTRY_DECL(gemm)
ENTRY_DECL(colsum)
ENTRY_DECL(relu)
ENTRY_DECL(relu_bwd)
ENTRY_DECL(relu6)
ENTRY_DECL(relu6_bwd)
ENTRY_DECL(add)
ENTRY_DECL(mse)
ENTRY_DECL(sgd)
ENTRY_DECL(conv_fwd)
ENTRY_DECL(conv_dgrad)
ENTRY_DECL(conv_wgrad)
ENTRY_DECL(dw_fwd)
ENTRY_DECL(dw_dgrad)
ENTRY_DECL(dw_wgrad)
ENTRY_DECL(bn_eval)
ENTRY_DECL(bn_stats)
ENTRY_DECL(bn_apply)
ENTRY_DECL(bn_bwd_reduce)
ENTRY_DECL(bn_bwd_dx)
ENTRY_DECL(maxpool)
ENTRY_DECL(avgpool)
ENTRY_DECL(avgpool_bwd)
ENTRY_DECL(ce)
ENTRY_DECL(gemm_bf16)
ENTRY_DECL(attention)
ENTRY_DECL(layernorm)
ENTRY_DECL(gelu)
ENTRY_DECL(add_bf16)
ENTRY_DECL(embed)
ENTRY_DECL(maxpool_bwd)
ENTRY_DECL(col2im)
ENTRY_DECL(layernorm_f32)
ENTRY_DECL(layernorm_f32_bwd)
ENTRY_DECL(attention_f32)
ENTRY_DECL(attention_f32_bwd_dq)
ENTRY_DECL(attention_f32_bwd_dkv)
