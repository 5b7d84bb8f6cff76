"""The offline profiler's classification (R16) and SM requirement (R17)
against the values the paper and the hardware limits fix (no GPU).

Pins:
  * the paper's worked throughputs: Conv2d at 89 % compute / 20 % memory is compute-
    bound, BN2d at 14 % / 80 % memory-bound; both under 60 % and no roofline -> unknown;
    ncu's 60 % threshold is strict;
  * the roofline ridge follows the pipe the kernel runs on: an fp32 1x1 conv of ResNet-50 at batch
    64 (~26 flop/B) is compute-bound on the FFMA ridge (11.4) but memory-bound on the 3xTF32
    tensor path (ridge 42.4) it actually takes;
  * sm_needed = ceil(num_blocks / blocks_per_sm) with blocks_per_sm the tightest of the thread,
    register and shared-memory limits; SURVEY §8(c).5's two worked examples, worked by
    hand from the sm_100 limits (2048 threads, 64 K registers, 32 CTAs, 228 KB shared memory,
    1 KB reserved per CTA)."""
import pytest

from paper_conf_eurosys_stratimk24_b200 import _lib as L, profiler as PR


def test_paper_worked_throughputs():
    assert PR.classify(89, 20) == L.CLS_C      # Conv2d
    assert PR.classify(14, 80) == L.CLS_M      # BN2d
    assert PR.classify(59, 40) == L.CLS_U      # both below 60 %, no roofline
    assert PR.classify(60, 60) == L.CLS_U      # "over 60%": strict
    assert PR.classify(61, 60.5) == L.CLS_C and PR.classify(60.5, 61) == L.CLS_M


def test_roofline_first():
    # roofline analysis takes precedence over the throughput percentages
    assert PR.classify(10, 90, flops=100, dram_bytes=1, ridge=11.4) == L.CLS_C
    assert PR.classify(90, 10, flops=1, dram_bytes=100, ridge=11.4) == L.CLS_M


def test_ridge_per_pipe():
    assert PR.RIDGE_FFMA == pytest.approx(148 * 128 * 2 * 1.965e9 / 6554.2e9, rel=1e-12)
    assert PR.RIDGE_FFMA == pytest.approx(11.36, abs=0.01)
    assert PR.RIDGE_TF32X3 == pytest.approx(1669.2e12 / 6 / 6554.2e9, rel=1e-12)
    assert PR.RIDGE_TF32X3 == pytest.approx(42.45, abs=0.01)
    # ResNet-50 b64 layer1 1x1 conv 64 -> 256 over 64*56*56 rows: 2MNK / 4(MK + KN + MN)
    M, N, K = 64 * 56 * 56, 256, 64
    ai = 2 * M * N * K / (4 * (M * K + K * N + M * N))
    assert 25 < ai < 26
    assert PR.classify(flops=2 * M * N * K, dram_bytes=4 * (M * K + K * N + M * N), ridge=PR.RIDGE_FFMA) == L.CLS_C
    assert PR.classify(flops=2 * M * N * K, dram_bytes=4 * (M * K + K * N + M * N), ridge=PR.RIDGE_TF32X3) == L.CLS_M
    assert PR.RIDGE_OF_PIPE[L.PIPE_TF32X3] == PR.RIDGE_TF32X3 and PR.RIDGE_OF_PIPE[L.PIPE_BF16] == PR.RIDGE_BF16


def test_sm_needed_worked_examples():
    # (a) grid 1000, 256 threads, 64 registers, 48 KB shared: threads 2048/256 = 8, registers
    # 65536/(64*256) = 4, shared 233472/(49152+1024) = 4.65 -> 4, CTAs 32 -> 4 per SM -> 250 SMs
    lim = PR.occupancy_limits(256, 64, 48 * 1024)
    assert lim == {"warps": 8, "registers": 4, "shared_mem": 4, "blocks": 32}
    assert PR.sm_needed_closed_form(1000, 256, 64, 48 * 1024) == 250
    # (b) grid 64, 128 threads, 32 registers, no shared memory: 16 (warps), 16 (registers) -> 4 SMs
    lim = PR.occupancy_limits(128, 32, 0)
    assert lim["warps"] == 16 and lim["registers"] == 16 and lim["blocks"] == 32
    assert PR.sm_needed_closed_form(64, 128, 32, 0) == 4


def test_occupancy_granularities():
    # registers are allocated per warp in units of 256: 33 registers cost as much as 40
    assert PR.occupancy_limits(256, 33, 0)["registers"] == PR.occupancy_limits(256, 40, 0)["registers"] == 6
    # a 1-thread CTA still takes a whole warp; the CTA limit (32) binds
    assert PR.blocks_per_sm_closed_form(1, 16, 0) == 32
    # shared memory: 128-byte granularity + 1 KB reserved per CTA; 227 KB is one CTA per SM
    assert PR.occupancy_limits(128, 32, 227 * 1024)["shared_mem"] == 1
    assert PR.occupancy_limits(128, 32, 100 * 1024 + 1)["shared_mem"] == 2
    # registers come from four 16 K sub-partitions: 9 warps of 112 registers (3584 per warp) fit 4
    # warps per partition = 16 per SM -> one 288-thread CTA, not the two 64 K / (9 x 3584) suggests
    # (measured: cudaOccupancyMaxActiveBlocksPerMultiprocessor = 1 for wgs_kernel at 109 registers)
    assert PR.occupancy_limits(288, 109, 98 * 1024)["registers"] == 1
    assert PR.occupancy_limits(256, 119, 98 * 1024)["registers"] == 2
    # a kernel that needs more SMs than the GPU has is never admitted beside the HP (L27, R5)
    assert PR.sm_needed_closed_form(296, 256, 119, 97 * 1024) == 148


def _ncu_tables():
    import csv
    import glob
    import os
    root = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles")
    for path in sorted(glob.glob(os.path.join(root, "*_ncu.csv"))):
        rows = list(csv.DictReader(open(path)))
        if rows and "occ_regs" in rows[0] and rows[0]["occ_regs"] not in ("", None):
            yield os.path.basename(path), rows


def test_occupancy_closed_form_matches_ncu():
    """R17 pinned to the hardware: for every launch of the committed per-op ncu tables (one solo
    launch per op on a B200, tools/ncu_times.sh with NCU_PROFILE=1), the closed-form limits from
    the launch's block size, registers per thread and shared memory equal ncu's
    launch__occupancy_limit_{warps,registers,blocks[,shared_mem]} -- the quantities P:863-868 names."""
    n = 0
    for name, rows in _ncu_tables():
        for r in rows:
            block, regs = int(float(r["block"])), int(float(r["regs"]))
            smem = None
            if r.get("smem_dyn") not in (None, "") and r.get("smem_static") not in (None, ""):
                smem = int(float(r["smem_dyn"])) + int(float(r["smem_static"]))
            lim = PR.occupancy_limits(block, regs, smem or 0)
            assert lim["warps"] == int(float(r["occ_warps"])), (name, r["label"])
            assert lim["registers"] == int(float(r["occ_regs"])), (name, r["label"], block, regs)
            assert lim["blocks"] == int(float(r["occ_blocks"])), (name, r["label"])
            if smem is not None:
                # ncu's shared-memory limit uses the carveout the driver configured for the launch,
                # never more than the full 228 KB the closed form assumes; the binding limit
                # (blocks_per_sm, what sm_needed divides by) agrees exactly
                assert lim["shared_mem"] >= int(float(r["occ_smem"])), (name, r["label"], smem)
                ncu_min = min(int(float(r[k])) for k in ("occ_warps", "occ_regs", "occ_blocks", "occ_smem"))
                assert min(lim.values()) == ncu_min, (name, r["label"], lim, ncu_min)
            n += 1
    if n == 0:
        pytest.skip("no committed ncu table carries the occupancy limits")
    assert n >= 100
