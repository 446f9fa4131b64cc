"""plgen — seeded synthetic input generators shared by the CUDA path and the oracle.

This module holds NO arithmetic of the method (no stage logic, no scheduling,
no solver).  It only draws the synthetic inputs the paper's workloads are made
of (§6.1) and packs them into the byte layouts both sides
read:

* ``dna``      — 2-bit packed DNA database / query with planted matches
                 (configs c2–c5).
* ``gaintab``  — the per-stage random-gain thresholds of the paper's gain model
                 (§6.1): the *distribution tables* the method
                 draws from, passed to both sides as input.
* ``arrivals`` — random arrival times (Poisson) as an input array.
* ``configs``  — the named configurations of BASELINE.json (c1..c5) and the
                 timing parameters of PAPER.md Table 1 (L218–L225).
"""
from . import arrivals, dna, gaintab, configs  # noqa: F401
