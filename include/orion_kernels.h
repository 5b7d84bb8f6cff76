/*
 * orion_kernels.h — the operator table of liborion: hand-written sm_100a kernels that an
 * orion_op names through orion_op.fn (part of the C ABI, see orion.h).
 *
 * The paper's operators are cuDNN/cuBLAS/PyTorch kernels of TorchVision models run in fp32
 * (P:888-899); here each is an explicit kernel with the PyTorch semantics written out in
 * oracle/model.py. Layouts in HBM: activations NHWC fp32, conv weights OHWI fp32
 * ([Cout][kh][kw][Cin/groups]), linear weights [out][in], labels int32. All pointers are device
 * pointers owned by the caller (torch tensors) and must stay alive until the op completes.
 *
 * Every kernel is deterministic and independent of the SM partition it runs in (no float
 * atomics, fixed reduction order, no SM-count-dependent tiling), so a client's outputs are
 * bitwise identical solo and collocated.
 *
 * Arg layouts: args[i] as listed (u64; floats as their fp32 bit pattern in the low 32 bits).
 */
#ifndef ORION_KERNELS_H
#define ORION_KERNELS_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum orion_fn {
  /* C[M,N] = op(A) op(B) (+ bias[N]); row-major; op = transpose if flag set.
     args: A, B, C, bias (0 = none), M, N, K, lda, ldb, ldc, flags (1 = A^T, 2 = B^T).
     y = x W^T + b (Linear fwd) is flags=2; dx = dy W is flags=0; dW = dy^T x is flags=1.
     args[11], args[12] = workspace, ws_bytes for the shape-selected K split (0 = no split); size
     from orion_gemm_workspace_bytes(M, N, K). */
  ORION_FN_GEMM = 0,
  /* Column sum: out[n] = sum_m A[m, n]  (bias gradient). args: A, out, M, N */
  ORION_FN_COLSUM = 1,
  /* y = max(x, 0). args: x, y, n */
  ORION_FN_RELU = 2,
  /* dx = dy * (x > 0). args: x, dy, dx, n */
  ORION_FN_RELU_BWD = 3,
  /* y = min(max(x, 0), 6). args: x, y, n */
  ORION_FN_RELU6 = 4,
  /* dx = dy * (0 < x < 6). args: x, dy, dx, n */
  ORION_FN_RELU6_BWD = 5,
  /* c = a + b. args: a, b, c, n */
  ORION_FN_ADD = 6,
  /* MSE loss mean((y-t)^2) and dy = 2(y-t)/n. args: y, t, loss (1 float), dy, n */
  ORION_FN_MSE = 7,
  /* SGD with momentum (torch semantics, dampening 0): v = mu v + g; p -= lr v. With v
     initialised to 0 the first step equals torch's v = g. mu = 0: p -= lr g (v unused).
     args: p, g, v, n, lr_bits, mu_bits */
  ORION_FN_SGD = 8,
  /* Conv2d forward, implicit GEMM, groups = 1, no bias. args: x, w, y, N, H, W, C, K(=Cout),
     R, S (kernel h, w), stride, pad, P, Q (out h, w), workspace, ws_bytes (split-K; 0 = no split;
     size from orion_gemm_workspace_bytes(N*P*Q, K, R*S*C)) */
  ORION_FN_CONV_FWD = 9,
  /* Conv2d backward data: dx[N,H,W,C] from dy[N,P,Q,K], w. args: dy, w, dx, N,H,W,C,K,R,S,stride,pad,P,Q,
     workspace, ws_bytes (orion_gemm_workspace_bytes(N*H*W, C, R*S*K)) */
  ORION_FN_CONV_DGRAD = 10,
  /* Conv2d backward weight: dw[K,R,S,C] from x, dy. args: x, dy, dw, N,H,W,C,K,R,S,stride,pad,P,Q,
     workspace, ws_bytes (orion_conv_wgrad_workspace_bytes(N, H, W, C, K, R, S, stride, pad)) */
  ORION_FN_CONV_WGRAD = 11,
  /* Depthwise 3x3 conv (groups = C): args as CONV_* with K = C */
  ORION_FN_DW_FWD = 12,
  ORION_FN_DW_DGRAD = 13,
  ORION_FN_DW_WGRAD = 14,
  /* BN eval: y = (x - rm) * rsqrt(rv + eps) * gamma + beta. args: x, y, gamma, beta, rm, rv, rows, C, eps_bits */
  ORION_FN_BN_EVAL = 15,
  /* BN train statistics (batch mean, biased var) + running-stat update (momentum, unbiased var).
     args: x, mean, invstd, rm, rv, rows, C, eps_bits, momentum_bits, workspace, ws_bytes */
  ORION_FN_BN_STATS = 16,
  /* BN train apply: y = (x - mean) * invstd * gamma + beta. args: x, y, gamma, beta, mean, invstd, rows, C */
  ORION_FN_BN_APPLY = 17,
  /* BN backward reduce: dgamma = sum dy*xhat, dbeta = sum dy. args: x, dy, mean, invstd, dgamma, dbeta,
     rows, C, workspace, ws_bytes */
  ORION_FN_BN_BWD_REDUCE = 18,
  /* BN backward dx = gamma*invstd/N (N dy - dbeta - xhat dgamma). args: x, dy, dx, gamma, mean, invstd,
     dgamma, dbeta, rows, C */
  ORION_FN_BN_BWD_DX = 19,
  /* MaxPool 3x3 stride 2 pad 1. args: x, y, N, H, W, C, P, Q */
  ORION_FN_MAXPOOL = 20,
  /* Global average pool [N,H,W,C] -> [N,C]. args: x, y, N, HW, C */
  ORION_FN_AVGPOOL = 21,
  /* Its backward: dx[n,hw,c] = dy[n,c] / HW. args: dy, dx, N, HW, C */
  ORION_FN_AVGPOOL_BWD = 22,
  /* Softmax cross entropy (mean over batch) and dz = (softmax - onehot)/B.
     args: z, labels(int32), loss (1 float), dz, B, classes */
  ORION_FN_CE = 23,
  /* ---- bf16 transformer operators (HP of BASELINE config 3: BERT-base inference as PyTorch
     eager runs a bfloat16 HuggingFace BertModel; readings R22, R29-R31). bf16 tensors
     are row-major, 16-byte aligned; arithmetic is fp32, each output rounded once (RNE).
     Linear: y[M,N] = x[M,K] W[N,K]^T + b[N] on tcgen05 (kind::f16, fp32 TMEM accumulator).
     args: x, W, y, b (0 = none), M, N, K. K % 8 == 0 (else ORION_E_INVAL). */
  ORION_FN_GEMM_BF16 = 24,
  /* Scaled dot-product attention without mask, one op: per batch b and head h,
     O = softmax(Q K^T / sqrt(d)) V over the head's d columns. q, k, v, o: [B, S, ld] with head h at
     columns h*d .. h*d+d-1. args: q, k, v, o, B, S, heads, d, ld. d == 64, S in {16, 32, 64, 128},
     ld % 8 == 0 (else ORION_E_INVAL). P is rounded to bf16 before P V (flash-style). */
  ORION_FN_ATTENTION = 25,
  /* LayerNorm over the last dim (biased variance): y = (x - mean) / sqrt(var + eps) * gamma + beta.
     args: x, y, gamma, beta, rows, C, eps_bits. C % 8 == 0, C <= 2048. */
  ORION_FN_LAYERNORM = 26,
  /* GELU, erf form: y = 0.5 x (1 + erf(x / sqrt 2)). args: x, y, n (n % 8 == 0) */
  ORION_FN_GELU = 27,
  /* bf16 residual add c = a + b. args: a, b, c, n (n % 8 == 0) */
  ORION_FN_ADD_BF16 = 28,
  /* Embedding sum: out[b, s, :] = word[ids[b, s]] + type[0] + pos[s] (token type 0, no padding).
     args: ids (int32 [B*S]), word [vocab, H], pos [>= S, H], type [>= 1, H], out [B, S, H], B, S, H,
     vocab. H % 8 == 0. Ids outside [0, vocab) are clamped into it. */
  ORION_FN_EMBED = 29,
  /* ---- fp32: MaxPool 3x3 / stride 2 / pad 1 backward. dx[n,h,w,c] = sum of dy over the windows
     whose first maximum (row-major window order) is x[n,h,w,c]. args: x, dy, dx, N, H, W, C, P, Q.
     C % 4 == 0; P, Q must be the forward's output size (else ORION_E_INVAL). */
  ORION_FN_MAXPOOL_BWD = 30,
  /* fp32 col2im (adjoint of im2col): dx[n,h,w,c] = sum over taps (r, s) with h = p*stride - pad + r,
     w = q*stride - pad + s of col[(n,p,q)][(r,s,c)]. With col = dy W (GEMM, W = OHWI weights as
     [K][R*S*C]) it is the data gradient of a strided convolution. args: col, dx, N, H, W, C, R, S,
     stride, pad, P, Q. C % 4 == 0; P, Q must be the conv's output size (else ORION_E_INVAL). */
  ORION_FN_COL2IM = 31,
  /* ---- fp32 Transformer-encoder training (BE of BASELINE config 4; reading R32): post-LN
     torch.nn.TransformerEncoderLayer. LayerNorm over the last dim (C % 128 == 0, C <= 512), saving
     the row mean and rstd = 1/sqrt(var + eps). args: x, y, gamma, beta, mean, rstd, rows, C, eps_bits */
  ORION_FN_LAYERNORM_F32 = 32,
  /* Its backward from the saved statistics: dx, dgamma = sum dy*xhat, dbeta = sum dy (column sums in
     fp64, CTA partials combined in order). args: x, dy, dx, gamma, mean, rstd, dgamma, dbeta, rows, C,
     workspace, ws_bytes (orion_layernorm_bwd_workspace_bytes(rows, C)) */
  ORION_FN_LAYERNORM_F32_BWD = 33,
  /* Attention forward, fp32: per batch b and head h, O = softmax(Q K^T / sqrt(d)) V over the head's
     d = 64 columns. q, k, v rows of stride ld_in (e.g. the packed [rows, 3d] in-projection), o of
     stride ld_out. S % 32 == 0, S <= 256. args: q, k, v, o, B, S, heads, d, ld_in, ld_out */
  ORION_FN_ATTENTION_F32 = 34,
  /* Attention backward, op 1: dQ = dS K / sqrt(d) with dS = P (dO V^T - rowsum(P dO V^T)); writes the
     per-row statistics (max, 1/sum, rowsum) to stats [B][heads][S][3] for op 2.
     args: q, k, v, dO, dq, stats, B, S, heads, d, ld_in, ld_out (q, k, v, dq of stride ld_in: gradients
     share their input's layout, e.g. the packed [rows, 3d] buffer; dO of stride ld_out) */
  ORION_FN_ATTENTION_F32_BWD_DQ = 35,
  /* Attention backward, op 2: dV = P^T dO, dK = dS^T Q / sqrt(d) from the stats of op 1.
     args: q, k, v, dO, stats, dk, dv, B, S, heads, d, ld_in, ld_out (dk, dv of stride ld_in, dO of ld_out) */
  ORION_FN_ATTENTION_F32_BWD_DKV = 36,
  ORION_FN_COUNT = 37
};

/* Number of table entries, and a stable name for each (for profiles and logs). */
int orion_kernel_count(void);
const char* orion_kernel_name(uint32_t fn);
/* Launch one operator directly on `cu_stream` (no scheduler; the "native" path, R20, and the
   offline profiler's solo runner). */
int orion_kernel_launch(uint32_t fn, const uint64_t* args, uint32_t nargs, void* cu_stream);
/* Launch geometry of an operator as it would launch: total CTAs and the occupancy-limited
   CTAs per SM (cudaOccupancyMaxActiveBlocksPerMultiprocessor), for sm_needed (R17). */
int orion_kernel_geometry(uint32_t fn, const uint64_t* args, uint32_t nargs, uint64_t* grid_ctas,
                          int32_t* blocks_per_sm, int32_t* threads_per_cta, int32_t* smem_bytes);
/* Which pipe an operator's arithmetic runs on, as launched (the roofline ridge of the profiler's
   classifier depends on it, reading R16 / P:838-847): */
enum orion_pipe {
  ORION_PIPE_FMA = 0,     /* FP32 FFMA / ALU / load-store (SIMT kernels) */
  ORION_PIPE_TF32X3 = 1,  /* tcgen05 kind::tf32, 3 MMAs per fp32 product (3xTF32) */
  ORION_PIPE_BF16 = 2     /* bf16 tensor pipe (tcgen05 kind::f16 or mma.sync bf16) */
};
/* Everything the offline profiler needs about one launch ("the number of blocks, the
   number of threads per block, the number of registers per thread, and the amount of shared memory
   that the kernel requires"), for the op as it would launch. Returns 0 or ORION_E_INVAL / E_CUDA. */
typedef struct {
  uint64_t grid_ctas;        /* total CTAs of the launch */
  int32_t threads_per_cta;
  int32_t regs_per_thread;   /* cudaFuncAttributes.numRegs */
  int32_t static_smem;       /* cudaFuncAttributes.sharedSizeBytes */
  int32_t dynamic_smem;      /* dynamic shared memory per CTA of this launch */
  int32_t blocks_per_sm;     /* cudaOccupancyMaxActiveBlocksPerMultiprocessor */
  int32_t pipe;              /* enum orion_pipe */
  char kernel[120];          /* the kernel the op launches (mangled device-function name, truncated) */
  int32_t launches;          /* kernels one launch of the op issues (2: split partials + ordered combine) */
} orion_kernel_info_t;
int orion_kernel_info(uint32_t fn, const uint64_t* args, uint32_t nargs, orion_kernel_info_t* out);
/* Workspace sizes (bytes) of the ops that split their reductions. Workspaces must be zeroed once
   at allocation; a client's ops may share one (they run in stream order; tickets self-reset). */
uint64_t orion_gemm_workspace_bytes(uint64_t M, uint64_t N, uint64_t K);
/* CONV_WGRAD's workspace: the tiled split-K need, or (few-input-channel stems, C <= 4) the
   per-CTA fp64 partials of the direct stem weight-gradient kernel, whichever is larger. */
uint64_t orion_conv_wgrad_workspace_bytes(uint64_t N, uint64_t H, uint64_t W, uint64_t C, uint64_t K, uint64_t R, uint64_t S,
                                          uint64_t stride, uint64_t pad);
uint64_t orion_bn_workspace_bytes(uint64_t rows, uint64_t C);
uint64_t orion_layernorm_bwd_workspace_bytes(uint64_t rows, uint64_t C);
uint64_t orion_dw_wgrad_workspace_bytes(uint64_t N, uint64_t C, uint64_t P, uint64_t Q);

#ifdef __cplusplus
}
#endif
#endif /* ORION_KERNELS_H */
