"""Host-core placement of one Orion instance per GPU (replicas only).

Every instance runs three busy-polling host threads: the scheduler (Listing 1 loop), the HP client
driver and the BE client driver (one more per extra BE client). Sharing a core between two of them
puts the OS scheduler's time slice (milliseconds) into the HP's tail latency, so each gets a core of
its own, chosen from the GPU's NUMA node when `nvidia-smi topo -m` names one, else from the
process's allowed cores in order. Fewer free cores than threads fails loudly (set
ORION_ALLOW_OVERSUBSCRIBE=1 to share cores round robin instead, with a warning in the result)."""
import os
import re
import subprocess


class PlacementError(RuntimeError):
    pass


def parse_cpu_list(s):
    """'0-3,8,10-11' -> [0, 1, 2, 3, 8, 10, 11]"""
    out = []
    for part in s.replace(" ", "").split(","):
        if not part:
            continue
        if "-" in part:
            a, b = part.split("-")
            out.extend(range(int(a), int(b) + 1))
        else:
            out.append(int(part))
    return out


def gpu_cpu_affinity(topo_text, gpu):
    """Cores `nvidia-smi topo -m` lists as the CPU affinity of GPU<gpu> (None if absent)."""
    lines = topo_text.splitlines()
    hdr = next((l for l in lines if "CPU Affinity" in l), None)
    if hdr is None:
        return None
    cols = re.split(r"\t+|\s{2,}", hdr.strip())
    try:
        ci = cols.index("CPU Affinity")
    except ValueError:
        return None
    for l in lines:
        f = re.split(r"\t+|\s{2,}", l.strip())
        if f and f[0] == f"GPU{gpu}" and len(f) > ci:
            try:
                return parse_cpu_list(f[ci])
            except ValueError:
                return None
    return None


def plan(local_rank, local_world, threads_per_instance, allowed, node_cpus=None, allow_oversubscribe=False):
    """Cores for instance `local_rank` of `local_world` on this host: a list of threads_per_instance
    distinct cores (scheduler first). node_cpus: this GPU's NUMA-local cores (preferred). Instances
    on one NUMA node split its cores in rank order; without NUMA information the allowed cores are
    split in rank order. Raises PlacementError when the cores do not suffice."""
    allowed = sorted(set(allowed))
    pool = [c for c in (node_cpus or []) if c in allowed]
    # instances sharing the node: assume ranks are spread evenly over the nodes the topology shows;
    # without it, every instance takes its slice of all allowed cores
    if len(pool) >= threads_per_instance and node_cpus:
        per = threads_per_instance
        # keep core 0 of the pool for the OS / launcher when there is room
        start = 1 if len(pool) > per else 0
        slot = local_rank % max(1, (len(pool) - start) // per)
        cores = pool[start + slot * per:start + (slot + 1) * per]
        if len(cores) == per:
            return cores, None
    need = local_world * threads_per_instance
    if len(allowed) >= need + 1:
        base = 1 + local_rank * threads_per_instance          # core 0 left to the OS / launcher
        return allowed[base:base + threads_per_instance], None
    if len(allowed) >= need:
        base = local_rank * threads_per_instance
        return allowed[base:base + threads_per_instance], None
    msg = (f"{len(allowed)} host cores for {local_world} Orion instance(s) x {threads_per_instance} busy-polling "
           f"threads: fewer than one core per thread")
    if not allow_oversubscribe:
        raise PlacementError(msg + " (set ORION_ALLOW_OVERSUBSCRIBE=1 to share cores)")
    cores = [allowed[(local_rank * threads_per_instance + i) % len(allowed)] for i in range(threads_per_instance)]
    return cores, "oversubscribed: " + msg


def for_this_process(local_rank, local_world, threads_per_instance):
    """plan() with this process's allowed cores and this GPU's NUMA affinity from nvidia-smi."""
    allowed = sorted(os.sched_getaffinity(0))
    node = None
    try:
        topo = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True, timeout=20).stdout
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        gpu = int(vis.split(",")[local_rank]) if vis else local_rank
        node = gpu_cpu_affinity(topo, gpu)
    except Exception:
        node = None
    return plan(local_rank, local_world, threads_per_instance, allowed, node,
                allow_oversubscribe=os.environ.get("ORION_ALLOW_OVERSUBSCRIBE") == "1")


def pin_current_thread(core):
    """Pin the calling thread (Linux: pid 0 = this thread) to one core; returns the previous mask."""
    prev = os.sched_getaffinity(0)
    if core is not None:
        os.sched_setaffinity(0, {core})
    return prev
