"""Arrival-time inputs (seeded) for the arrival processes of the executor.

PAPER.md §2.1: items arrive at a fixed rate rho0 (a(r) = r * tau0; the default, no
array needed).  §7: Poisson arrivals are "a reasonable generalization of the fixed
arrival rate".  The random arrival times are an INPUT handed to both the
CUDA path and the oracle (int64 per root, relative to the start of the root's stream), so
neither side draws them.

Poisson: a(0) = 0, a(r) = a(r-1) + round(Exp(mean tau0)) per stream (integer time units;
gaps of 0 are simultaneous arrivals).
"""
from __future__ import annotations

import numpy as np


def poisson(seed: int, stream_sizes, tau0: float) -> np.ndarray:
    rng = np.random.default_rng(np.random.PCG64(seed ^ 0xA221A1))
    out = []
    for n in stream_sizes:
        if n == 0:
            continue
        gaps = np.rint(rng.exponential(tau0, size=n)).astype(np.int64)
        gaps[0] = 0
        out.append(np.cumsum(gaps))
    return np.concatenate(out) if out else np.zeros(0, dtype=np.int64)


def stream_sizes(n_roots_total: int, n_streams: int):
    return [((s + 1) * n_roots_total) // n_streams - (s * n_roots_total) // n_streams for s in range(n_streams)]
