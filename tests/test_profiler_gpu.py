"""R17 on the GPU: for every kernel op of the configs' clients, the closed-form blocks_per_sm
(profiler.occupancy_limits from the kernel's threads, registers and shared memory)
equals the CUDA occupancy API's, and -- where the committed per-op ncu capture carries them --
ncu's own launch__occupancy_limit_{warps,registers,shared_mem,blocks}. Also checks that the pipe
each op reports is the one its roofline ridge assumes (tensor-core kernels report a tensor pipe)."""
import csv
import os

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

if torch.cuda.is_available():
    import bench
    from paper_conf_eurosys_stratimk24_b200 import _lib as L, profiler as PR
    from paper_conf_eurosys_stratimk24_b200.runtime import kernel_info


def _ncu_rows(cfg, client, base):
    p = os.path.join(ROOT, "profiles", f"{cfg}_{client}_ncu.csv")
    if not os.path.exists(p):
        return {}
    out = {}
    for r in csv.DictReader(open(p)):
        if r.get("occ_warps") not in (None, ""):
            out[int(r["kernel_id"]) - base] = r
    return out


@pytest.mark.parametrize("cfg,client", [("rn50_mnv2", "hp"), ("rn50_mnv2", "be"), ("bert_rn50", "hp"), ("rn101_enc", "be")])
def test_closed_form_occupancy_matches_cuda_and_ncu(cfg, client):
    torch.cuda.set_device(0)
    g = bench.build_client(cfg, client)
    ncu = _ncu_rows(cfg, client, 10000 if client == "be" else 0)
    checked_ncu = 0
    pipes = {}
    for i, fn, args, lab in g.kernel_ops():
        info = kernel_info(fn, args)
        smem = info["static_smem"] + info["dynamic_smem"]
        cf = PR.blocks_per_sm_closed_form(info["threads_per_cta"], info["regs_per_thread"], smem)
        assert cf == info["blocks_per_sm"], (lab, fn, info, PR.occupancy_limits(info["threads_per_cta"], info["regs_per_thread"], smem))
        pipes.setdefault(fn, set()).add(info["pipe"])
        r = ncu.get(i)
        # (a committed row describes the launch as it was built then: compare only rows whose grid,
        # block size and registers are this build's)
        if r is not None and int(float(r["grid"])) == info["grid_ctas"] and int(float(r["block"])) == info["threads_per_cta"] \
                and int(float(r["regs"])) == info["regs_per_thread"]:
            lim = PR.occupancy_limits(info["threads_per_cta"], info["regs_per_thread"], smem)
            assert int(float(r["occ_warps"])) == lim["warps"], (lab, r)
            assert int(float(r["occ_regs"])) == lim["registers"], (lab, r)
            # ncu's shared-memory limit follows the carveout the driver configured for the launch
            # (<= the full 228 KB the closed form assumes); the binding limit agrees exactly
            assert int(float(r["occ_smem"])) <= lim["shared_mem"], (lab, r)
            ncu_min = min(int(float(r[k])) for k in ("occ_warps", "occ_regs", "occ_blocks", "occ_smem"))
            assert ncu_min == min(lim.values()) == info["blocks_per_sm"], (lab, r, lim)
            checked_ncu += 1
    if ncu:
        assert checked_ncu >= len(ncu) // 2, f"committed ncu table mostly stale ({checked_ncu} of {len(ncu)} rows match this build)"
    # tensor-core operators report a tensor pipe; elementwise ones the FMA/ALU pipe
    for fn in ("relu", "relu6", "bn_apply", "bn_stats", "add", "layernorm", "gelu"):
        if fn in pipes:
            assert pipes[fn] == {L.PIPE_FMA}, (fn, pipes[fn])
    if "gemm_bf16" in pipes:
        assert pipes["gemm_bf16"] == {L.PIPE_BF16}
    if cfg == "rn50_mnv2" and client == "hp":
        assert L.PIPE_TF32X3 in pipes["conv_fwd"] and L.PIPE_TF32X3 in pipes["gemm"]
    print(f"{cfg}/{client}: {len(g.kernel_ops())} ops, ncu-checked {checked_ncu}")
