"""Offline workload profiler (§5.2), B200 edition.

For every operator of a client's op list it produces the profile row Orion's policy consumes:
  * dur_ns     — solo execution time, median of CUDA-event-timed solo launches;
  * sm_needed  — ceil(num_blocks / blocks_per_sm) with blocks_per_sm the occupancy limit of the
                 kernel as launched (reading R17);
  * cls        — compute (C) / memory (M) / unknown (U) (reading R16): roofline first
                 (algorithmic FLOPs / measured DRAM bytes vs the ridge of the pipe the kernel uses),
                 else >60% compute or memory throughput from ncu, else unknown.
ncu counters come from tools/profile/ncu_profile.py (run on the GPU box; CSV committed under
profiles/). Without a capture the classifier falls back to the analytic roofline of the op
(algorithmic bytes and FLOPs computed here from the op's shape), and says so in the row.
"""
import csv
import math
import os

import torch

from . import _lib as L
from .runtime import kernel_launch, kernel_geometry, kernel_info

# B200 peaks (MEASURED_PEAKS.json; FFMA peak derived: 148 SMs x 128 FMA x 2 x 1.965 GHz)
HBM_GBS = 6554.2
FFMA_TFLOPS = 148 * 128 * 2 * 1.965e9 / 1e12
RIDGE_FFMA = FFMA_TFLOPS * 1e12 / (HBM_GBS * 1e9)   # flop per DRAM byte (11.4)
BF16_TFLOPS = 1669.2                                  # dense bf16 tensor pipe (MEASURED_PEAKS.json)
RIDGE_BF16 = BF16_TFLOPS * 1e12 / (HBM_GBS * 1e9)
# fp32 GEMM / conv on tcgen05 kind::tf32 with three MMAs per product (3xTF32): tf32 dense = bf16 x
# the guide's nominal 1/2, so the algorithmic fp32 ceiling is bf16 / 6 -> ridge 42.4
TF32X3_TFLOPS = BF16_TFLOPS / 6.0
RIDGE_TF32X3 = TF32X3_TFLOPS * 1e12 / (HBM_GBS * 1e9)
RIDGE_OF_PIPE = {L.PIPE_FMA: RIDGE_FFMA, L.PIPE_TF32X3: RIDGE_TF32X3, L.PIPE_BF16: RIDGE_BF16}

# sm_100 per-SM limits for the closed-form occupancy (R17): threads, warps, CTAs,
# registers (64 K per SM in four 16 K sub-partitions, each warp's allocated from one of them in
# units of 256), shared memory (228 KB per SM, 1 KB reserved per CTA, 128-byte granularity)
SM_MAX_THREADS, SM_MAX_WARPS, SM_MAX_CTAS = 2048, 64, 32
SM_REGS, SM_PARTITIONS, REG_ALLOC_UNIT = 65536, 4, 256
SM_SMEM, CTA_SMEM_RESERVED, SMEM_ALLOC_UNIT = 233472, 1024, 128


def op_work(fn, a):
    """Algorithmic FLOPs and compulsory DRAM bytes of one op (each input read once, each output
    written once; fp32). The per-op numbers DESIGN.md §7 tabulates."""
    f = L.kernel_names()[fn] if isinstance(fn, int) else fn
    if f == "gemm":
        M, N, K = a[4], a[5], a[6]
        return 2 * M * N * K, 4 * (M * K + K * N + M * N + (N if a[3] else 0))
    if f in ("conv_fwd", "conv_dgrad", "conv_wgrad"):
        n, h, w, c, k, r, s, st, pad, p, q = a[3:14]
        return 2 * n * p * q * k * r * s * c, 4 * (n * h * w * c + k * r * s * c + n * p * q * k)
    if f in ("dw_fwd", "dw_dgrad", "dw_wgrad"):
        n, h, w, c, k, r, s, st, pad, p, q = a[3:14]
        return 2 * n * p * q * c * 9, 4 * (n * h * w * c + 9 * c + n * p * q * c)
    if f in ("relu", "relu6"):
        return a[2], 8 * a[2]
    if f in ("relu_bwd", "relu6_bwd", "add"):
        return a[3], 12 * a[3]
    if f == "bn_eval":
        return 2 * a[6] * a[7], 8 * a[6] * a[7]
    if f == "bn_stats":
        return 3 * a[5] * a[6], 4 * a[5] * a[6]
    if f == "bn_apply":
        return 2 * a[6] * a[7], 8 * a[6] * a[7]
    if f == "bn_bwd_reduce":
        return 4 * a[6] * a[7], 8 * a[6] * a[7]
    if f == "bn_bwd_dx":
        return 6 * a[8] * a[9], 12 * a[8] * a[9]
    if f == "maxpool":
        n, h, w, c, p, q = a[2:8]
        return 9 * n * p * q * c, 4 * (n * h * w * c + n * p * q * c)
    if f == "avgpool":
        return a[2] * a[3] * a[4], 4 * (a[2] * a[3] * a[4] + a[2] * a[4])
    if f == "avgpool_bwd":
        return a[2] * a[3] * a[4], 4 * (a[2] * a[3] * a[4] + a[2] * a[4])
    if f == "ce":
        return 5 * a[4] * a[5], 4 * 2 * a[4] * a[5]
    if f == "mse":
        return 3 * a[4], 12 * a[4]
    if f == "sgd":
        return 3 * a[3], (20 if a[5] else 12) * a[3]
    if f == "colsum":
        return a[2] * a[3], 4 * (a[2] * a[3] + a[3])
    # bf16 transformer ops: 2 bytes per element
    if f == "gemm_bf16":
        M, N, K = a[4], a[5], a[6]
        return 2 * M * N * K, 2 * (M * K + K * N + M * N + (N if a[3] else 0))
    if f == "attention":
        B, S, H, d = a[4], a[5], a[6], a[7]
        return 4 * B * H * S * S * d + 5 * B * H * S * S, 2 * 4 * B * S * H * d
    if f == "layernorm":
        return 8 * a[4] * a[5], 2 * (2 * a[4] * a[5] + 2 * a[5])
    if f == "gelu":
        return 8 * a[2], 4 * a[2]
    if f == "add_bf16":
        return a[3], 6 * a[3]
    if f == "embed":
        B, S, H = a[5], a[6], a[7]
        return 2 * B * S * H, 2 * (2 * B * S * H + S * H + H) + 4 * B * S
    if f == "col2im":
        n, h, w, c, r, s_, st, pad, p, q = a[2:12]
        return n * p * q * r * s_ * c, 4 * (n * p * q * r * s_ * c + n * h * w * c)
    if f == "layernorm_f32":
        return 8 * a[6] * a[7], 4 * (2 * a[6] * a[7] + 2 * a[6] + 2 * a[7])
    if f == "layernorm_f32_bwd":
        return 12 * a[8] * a[9], 4 * (3 * a[8] * a[9] + 2 * a[8] + 3 * a[9])
    if f in ("attention_f32", "attention_f32_bwd_dq", "attention_f32_bwd_dkv"):
        k0 = {"attention_f32": 4, "attention_f32_bwd_dq": 6, "attention_f32_bwd_dkv": 7}[f]
        B, S, H, d = a[k0], a[k0 + 1], a[k0 + 2], a[k0 + 3]
        mul = {"attention_f32": (4, 4), "attention_f32_bwd_dq": (6, 5), "attention_f32_bwd_dkv": (8, 6)}[f]
        return mul[0] * B * H * S * S * d, 4 * mul[1] * B * S * H * d
    if f == "maxpool_bwd":
        n, h, w, c, p, q = a[3:9]
        return 9 * n * p * q * c, 4 * (2 * n * h * w * c + n * p * q * c)
    return 0, 0


def classify(c_pct=None, m_pct=None, flops=0, dram_bytes=0, ridge=RIDGE_FFMA):
    """R16. (1) roofline when defined: C iff arithmetic intensity >= ridge; (2) else >60% compute or
    memory throughput (ncu's own threshold): C iff c >= m; (3) else unknown."""
    if flops > 0 and dram_bytes > 0:
        return L.CLS_C if flops / dram_bytes >= ridge else L.CLS_M
    if c_pct is not None and m_pct is not None and (c_pct > 60 or m_pct > 60):
        return L.CLS_C if c_pct >= m_pct else L.CLS_M
    return L.CLS_U


def occupancy_limits(threads, regs, smem):
    """blocks_per_sm of a kernel from its launch resources, limit by limit ("limited by
    the number of threads, the number of registers, or the amount of shared memory"); the same
    quantities ncu reports as launch__occupancy_limit_{warps,registers,shared_mem,blocks}."""
    warps = -(-threads // 32)
    lim_warps = SM_MAX_WARPS // warps
    per_warp = -(-(regs * 32) // REG_ALLOC_UNIT) * REG_ALLOC_UNIT
    warps_by_regs = (SM_REGS // SM_PARTITIONS // per_warp) * SM_PARTITIONS if regs > 0 else SM_MAX_WARPS
    lim_regs = warps_by_regs // warps
    per_cta = -(-smem // SMEM_ALLOC_UNIT) * SMEM_ALLOC_UNIT + CTA_SMEM_RESERVED
    lim_smem = min(SM_SMEM // per_cta, SM_MAX_CTAS)   # (ncu reports the block cap for smem-free kernels)
    return {"warps": lim_warps, "registers": lim_regs, "shared_mem": lim_smem, "blocks": SM_MAX_CTAS}


def blocks_per_sm_closed_form(threads, regs, smem):
    return min(occupancy_limits(threads, regs, smem).values())


def sm_needed_closed_form(num_blocks, threads, regs, smem):
    """sm_needed = ceil(num_blocks / blocks_per_sm)."""
    return int(math.ceil(num_blocks / max(blocks_per_sm_closed_form(threads, regs, smem), 1)))


def sm_needed(fn, args, num_sms=148):
    """R17 on the op as launched: the occupancy API's blocks_per_sm (== the closed form above,
    cross-checked on the GPU by tests/test_profiler_gpu.py)."""
    grid, bps, _, _ = kernel_geometry(fn, args)
    return int(math.ceil(grid / max(bps, 1)))


def ridge_of(fn, args):
    """Roofline ridge (flop per DRAM byte) of the pipe the op's kernel runs on as launched."""
    return RIDGE_OF_PIPE[kernel_info(fn, args)["pipe"]]


def time_ops(graph, reps=10, warmup=2, stream=None):
    """Median solo duration (ns) of every kernel op in the graph, each timed alone with CUDA events
    on the launching stream (per-kernel execution time)."""
    s = stream or torch.cuda.Stream()
    out = {}
    kops = graph.kernel_ops()
    with torch.cuda.stream(s):
        for i, fn, args, lab in kops:          # warm everything once (first-touch, module load)
            for _ in range(warmup):
                kernel_launch(fn, args, s.cuda_stream)
        torch.cuda.synchronize()
        for i, fn, args, lab in kops:
            ts = []
            for _ in range(reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                kernel_launch(fn, args, s.cuda_stream)
                e1.record(s)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e6)
            ts.sort()
            out[i] = int(ts[len(ts) // 2])
    return out


def load_ncu_csv(path):
    """{kernel_id: (c_pct, m_pct, dram_bytes, dur_ns)} from tools/profile/ncu_summarize.py's CSV
    (one solo launch per op under ncu: sm__throughput, gpu__compute_memory_throughput, DRAM bytes,
    gpu__time_duration)."""
    if not path or not os.path.exists(path):
        return {}
    rows = {}
    with open(path) as f:
        for r in csv.DictReader(f):
            rows[int(r["kernel_id"])] = (float(r["sm_pct"]), float(r["mem_pct"]), float(r["dram_bytes"]), float(r["dur_ns"]))
    return rows


def build_profiles(graph, kid_base=0, reps=10, ncu_csv=None):
    """Profile table {kernel_id: (cls, sm_needed, dur_ns)} + rows for the CSV."""
    durs = time_ops(graph, reps=reps)
    ncu = load_ncu_csv(ncu_csv)
    table, rows = {}, []
    for i, fn, args, lab in graph.kernel_ops():
        kid = kid_base + i
        flops, nbytes = op_work(fn, args)
        dur = durs[i]
        if kid in ncu:
            c, m, dram, ndur = ncu[kid]
            # arithmetic intensity over max(measured DRAM bytes, compulsory bytes): on B200 the 126 MB
            # L2 often holds an op's inputs, and DRAM bytes alone would call a memory-bound op
            # compute-bound (DESIGN.md §3 R16)
            cls = classify(c, m, flops, max(dram, nbytes), ridge_of(fn, args))
            dur = int(ndur) if ndur > 0 else dur   # device time of the kernel alone
            src = "ncu"
        else:
            cls = classify(None, None, flops, nbytes, ridge_of(fn, args))
            src = "analytic"
        sm = sm_needed(fn, args)
        table[kid] = (cls, sm, dur)
        rows.append(dict(kernel_id=kid, label=lab, fn=fn, cls="UCM"[cls], sm_needed=sm, dur_ns=dur,
                         flops=flops, bytes=nbytes, source=src))
    return table, rows


def write_profile_csv(path, rows):
    os.makedirs(os.path.dirname(path) or ".", exist_ok=True)
    with open(path, "w", newline="") as f:
        w = csv.DictWriter(f, fieldnames=list(rows[0].keys()))
        w.writeheader()
        w.writerows(rows)


def request_latency(run_once, n=100):
    """Median solo HP request latency (R9): run_once() returns one request's latency ns."""
    lats = sorted(run_once() for _ in range(n))
    return lats[len(lats) // 2]
