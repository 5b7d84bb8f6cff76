// The operator table (orion_kernels.h) and its direct-launch / geometry entry points.
#include "common.cuh"

#define E(fn, name, nargs) {#fn, nargs, name##_geom, name##_launch}
const KernelEntry g_kernels[ORION_FN_COUNT] = {
    E(gemm, gemm, 13),
    E(colsum, colsum, 4),
    E(relu, relu, 3),
    E(relu_bwd, relu_bwd, 4),
    E(relu6, relu6, 3),
    E(relu6_bwd, relu6_bwd, 4),
    E(add, add, 4),
    E(mse, mse, 6),
    E(sgd, sgd, 6),
    E(conv_fwd, conv_fwd, 16),
    E(conv_dgrad, conv_dgrad, 16),
    E(conv_wgrad, conv_wgrad, 16),
    E(dw_fwd, dw_fwd, 14),
    E(dw_dgrad, dw_dgrad, 14),
    E(dw_wgrad, dw_wgrad, 16),
    E(bn_eval, bn_eval, 9),
    E(bn_stats, bn_stats, 11),
    E(bn_apply, bn_apply, 8),
    E(bn_bwd_reduce, bn_bwd_reduce, 10),
    E(bn_bwd_dx, bn_bwd_dx, 10),
    E(maxpool, maxpool, 8),
    E(avgpool, avgpool, 5),
    E(avgpool_bwd, avgpool_bwd, 5),
    E(ce, ce, 7),
    E(gemm_bf16, gemm_bf16, 7),
    E(attention, attention, 9),
    E(layernorm, layernorm, 7),
    E(gelu, gelu, 3),
    E(add_bf16, add_bf16, 4),
    E(embed, embed, 9),
    E(maxpool_bwd, maxpool_bwd, 9),
    E(col2im, col2im, 12),
    E(layernorm_f32, layernorm_f32, 9),
    E(layernorm_f32_bwd, layernorm_f32_bwd, 12),
    E(attention_f32, attention_f32, 10),
    E(attention_f32_bwd_dq, attention_f32_bwd_dq, 12),
    E(attention_f32_bwd_dkv, attention_f32_bwd_dkv, 13),
};
#undef E

int kernel_launch_sig(uint32_t fn, const uint64_t* args, uint32_t nargs, OrionSig sig, cudaStream_t s, unsigned long long* ctas_out) {
  if (fn >= ORION_FN_COUNT || args == nullptr) return ORION_E_INVAL;
  const KernelEntry& e = g_kernels[fn];
  if ((int)nargs < e.nargs) return ORION_E_INVAL;
  LaunchGeom g;
  int r = e.geom(args, &g);
  if (r) return r;
  if (ctas_out) *ctas_out = g.signal_ctas();
  if (sig.ticket) sig.target += g.signal_ctas();
  return e.launch(args, g, sig, s);
}

extern "C" {

int orion_kernel_count(void) { return ORION_FN_COUNT; }

const char* orion_kernel_name(uint32_t fn) { return fn < ORION_FN_COUNT ? g_kernels[fn].name : "?"; }

int orion_kernel_launch(uint32_t fn, const uint64_t* args, uint32_t nargs, void* cu_stream) {
  OrionSig none{nullptr, nullptr, 0, 0};
  return kernel_launch_sig(fn, args, nargs, none, (cudaStream_t)cu_stream, nullptr);
}

int orion_kernel_geometry(uint32_t fn, const uint64_t* args, uint32_t nargs, uint64_t* grid_ctas, int32_t* blocks_per_sm,
                          int32_t* threads_per_cta, int32_t* smem_bytes) {
  if (fn >= ORION_FN_COUNT || args == nullptr) return ORION_E_INVAL;
  const KernelEntry& e = g_kernels[fn];
  if ((int)nargs < e.nargs) return ORION_E_INVAL;
  LaunchGeom g;
  int r = e.geom(args, &g);
  if (r) return r;
  int threads = (int)(g.block.x * g.block.y * g.block.z);
  if (grid_ctas) *grid_ctas = g.ctas();
  if (threads_per_cta) *threads_per_cta = threads;
  if (smem_bytes) *smem_bytes = g.smem;
  if (blocks_per_sm) {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, g.func, threads, g.smem) != cudaSuccess) return ORION_E_CUDA;
    *blocks_per_sm = b;
  }
  return 0;
}

int orion_kernel_info(uint32_t fn, const uint64_t* args, uint32_t nargs, orion_kernel_info_t* out) {
  if (fn >= ORION_FN_COUNT || args == nullptr || out == nullptr) return ORION_E_INVAL;
  const KernelEntry& e = g_kernels[fn];
  if ((int)nargs < e.nargs) return ORION_E_INVAL;
  LaunchGeom g;
  int r = e.geom(args, &g);
  if (r) return r;
  cudaFuncAttributes fa;
  if (cudaFuncGetAttributes(&fa, g.func) != cudaSuccess) { (void)cudaGetLastError(); return ORION_E_CUDA; }
  out->grid_ctas = g.ctas();
  out->threads_per_cta = (int32_t)(g.block.x * g.block.y * g.block.z);
  out->regs_per_thread = fa.numRegs;
  out->static_smem = (int32_t)fa.sharedSizeBytes;
  out->dynamic_smem = g.smem;
  out->pipe = g.pipe;
  out->launches = g.sig_ctas ? 2 : 1;
  int b = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, g.func, out->threads_per_cta, g.smem) != cudaSuccess) {
    (void)cudaGetLastError();
    return ORION_E_CUDA;
  }
  out->blocks_per_sm = b;
  const char* nm = nullptr;
  out->kernel[0] = 0;
  if (cudaFuncGetName(&nm, g.func) == cudaSuccess && nm) {
    size_t i = 0;
    for (; nm[i] && i + 1 < sizeof(out->kernel); i++) out->kernel[i] = nm[i];
    out->kernel[i] = 0;
  } else {
    (void)cudaGetLastError();
  }
  return 0;
}

}  // extern "C"
