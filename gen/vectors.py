"""Seeded dense vectors."""
from __future__ import annotations

import numpy as np
import torch


def uniform_vector(n: int, seed: int, lo: float = -1.0, hi: float = 1.0) -> torch.Tensor:
    """float64 U[lo, hi) (numpy PCG64, seed) as a CPU tensor."""
    rng = np.random.default_rng(seed)
    return torch.from_numpy(lo + (hi - lo) * rng.random(n))


def integer_vector(n: int, seed: int, lo: int = -3, hi: int = 3) -> torch.Tensor:
    """float64 integers uniform in {lo..hi} as a CPU tensor."""
    rng = np.random.default_rng(seed)
    return torch.from_numpy(rng.integers(lo, hi + 1, size=n).astype(np.float64))
