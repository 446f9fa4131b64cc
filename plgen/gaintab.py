"""Gain-distribution tables for the paper's random-gain pipeline model.

PAPER.md §6.1: "for each input, nodes 0, 2, and 3 produce one output with
probability g_i or 0 otherwise ... the number of outputs per input is Poisson
with mean g_i, censored at the upper limit u" (node 1).

The randomness itself is a counter-based hash each side implements on its own
(DESIGN.md "Readings" R-RNG); the *distribution* is handed to both sides as a
table of unsigned 64-bit thresholds, computed here once:

* Bernoulli(g):           thr = min(floor(g * 2^64), 2^64 - 1)
                          -> keep iff h < thr
* min(Poisson(lam), u):   thr_k = min(floor(CDF_lam(k) * 2^64), 2^64 - 1), k < u
                          -> count = #{k < u : h >= thr_k}

The floor of a double times 2^64 is taken exactly with ``fractions.Fraction``
(no rounding), so the table is bit-reproducible.
"""
from __future__ import annotations

import math
from fractions import Fraction

U64_MAX = (1 << 64) - 1


def prob_to_u64(p: float) -> int:
    if not (0.0 <= p <= 1.0):
        raise ValueError(f"probability out of range: {p}")
    return min(int(Fraction(p) * (1 << 64)), U64_MAX)


def poisson_cdf(lam: float, k: int) -> float:
    """CDF of Poisson(lam) at k, summed term by term in double precision."""
    term = math.exp(-lam)
    acc = term
    for j in range(1, k + 1):
        term *= lam / j
        acc += term
    return min(acc, 1.0)


def bernoulli_table(g: float) -> list:
    return [prob_to_u64(g)]


def poisson_capped_table(lam: float, u: int) -> list:
    return [prob_to_u64(poisson_cdf(lam, k)) for k in range(u)]
