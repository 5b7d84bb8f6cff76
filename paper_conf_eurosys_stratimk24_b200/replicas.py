"""Multi-GPU = independent replicas ("a separate instance of Orion runs per GPU
device"). Each rank runs its own Orion instance and workload on its own GPU; torch.distributed
(gloo) carries only the control plane: a barrier around the timed window and the gather of the
per-rank numbers. No collective touches the data path."""
import torch.distributed as dist


def init_from_env():
    """(rank, world, local_rank) from torchrun's environment; initialises gloo when world > 1."""
    import os
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if world > 1 and not dist.is_initialized():
        dist.init_process_group("gloo")
    return rank, world, local


def barrier():
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()


def gather(obj):
    """All ranks' objects, in rank order (a single-element list without torch.distributed)."""
    if not (dist.is_initialized() and dist.get_world_size() > 1):
        return [obj]
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, obj)
    return out


def aggregate(per_rank, steps):
    """Whole-job numbers from per-rank dicts {be_col, be_ded, win_ms, p99, p99d, p50, p50d, be_n}:
    throughput is summed over replicas (weak scaling: per-GPU work fixed), time is the max over
    ranks, HP tail latency is reported per rank and as the worst rank."""
    return {
        "value": sum(r["be_col"] for r in per_rank),
        "be_dedicated": sum(r["be_ded"] for r in per_rank),
        "ms_per_step": max(r["win_ms"] for r in per_rank) / max(steps, 1),
        "hp_p99_ratio_max": max(r["p99"] / r["p99d"] for r in per_rank),
        "hp_p99_ratio_per_rank": [r["p99"] / r["p99d"] for r in per_rank],
        "be_iterations": sum(r["be_n"] for r in per_rank),
    }
