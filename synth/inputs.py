"""Seeded input generators. No scheduling or model arithmetic lives here: only
draws from named distributions, so both the oracle and the CUDA path can consume the same bytes.

Seeds: weights seed 0; HP inputs seed 1 (request r uses sub-stream r);
BE data seed 2 (8 pre-staged batches cycled); arrivals seed 3 + 1000 * gpu_index.
"""
import math

import numpy as np
import torch

WEIGHT_SEED, HP_SEED, BE_SEED, ARRIVAL_SEED = 0, 1, 2, 3


def _gen(seed):
    g = torch.Generator(device="cpu")
    g.manual_seed(int(seed) & 0x7FFFFFFFFFFFFFFF)
    return g


def make_params(spec, seed=WEIGHT_SEED):
    """spec: ordered [(name, shape, init)], init one of
    ("uniform_fan_in", fan_in)  U(-1/sqrt(fan_in), 1/sqrt(fan_in))   (torch Linear default)
    ("kaiming_fan_out", fan_out) N(0, 2/fan_out)                       (torchvision conv init)
    ("normal", std) | ("uniform", lo, hi) | ("const", v).
    Every tensor is drawn from its own sub-stream (seed, index) so specs can be extended."""
    out = {}
    for i, (name, shape, init) in enumerate(spec):
        g = _gen(seed * 1_000_003 + i)
        kind = init[0]
        if kind == "uniform_fan_in":
            b = 1.0 / math.sqrt(init[1])
            t = (torch.rand(shape, generator=g, dtype=torch.float32) * 2 - 1) * b
        elif kind == "kaiming_fan_out":
            t = torch.randn(shape, generator=g, dtype=torch.float32) * math.sqrt(2.0 / init[1])
        elif kind == "normal":
            t = torch.randn(shape, generator=g, dtype=torch.float32) * init[1]
        elif kind == "uniform":
            t = init[1] + torch.rand(shape, generator=g, dtype=torch.float32) * (init[2] - init[1])
        elif kind == "const":
            t = torch.full(shape, float(init[1]), dtype=torch.float32)
        else:
            raise ValueError(kind)
        out[name] = t.contiguous()
    return out


def normal(shape, seed, sub=0):
    """N(0,1) fp32 tensor from sub-stream `sub` of `seed` (images NHWC, MLP inputs, targets)."""
    return torch.randn(shape, generator=_gen(seed * 1_000_003 + 7_919 * (sub + 1)), dtype=torch.float32)


def labels(n, num_classes, seed, sub=0):
    """Class labels U[0, num_classes) as int32."""
    g = _gen(seed * 1_000_003 + 104_729 * (sub + 1))
    return torch.randint(0, num_classes, (n,), generator=g, dtype=torch.int64).to(torch.int32)


def poisson_arrivals_ns(rate_rps, n, seed=ARRIVAL_SEED, gpu_index=0):
    """Open-loop Poisson arrivals: n scheduled arrival offsets (ns from start), exponential
    inter-arrival times with mean 1/rate (Table 3 rates; reading R21)."""
    rng = np.random.Generator(np.random.PCG64(seed + 1000 * gpu_index))
    gaps = rng.exponential(1.0 / rate_rps, size=n)
    return (np.cumsum(gaps) * 1e9).astype(np.int64)


def uniform_arrivals_ns(rate_rps, n):
    return (np.arange(1, n + 1) * (1e9 / rate_rps)).astype(np.int64)


def token_ids(shape, vocab, seed, sub=0):
    """Token ids U[0, vocab) as int32 (BERT inputs; token type 0, no padding: reading R22)."""
    g = _gen(seed * 1_000_003 + 15_485_863 * (sub + 1))
    return torch.randint(0, vocab, shape, generator=g, dtype=torch.int64).to(torch.int32)
