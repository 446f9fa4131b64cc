"""Statistical pins against the paper's own simulation statements .

P9 "the active fractions measured in the simulator closely matched those
    predicted by the optimizer": FIXED_WAIT within 1% of Fig. 1's T; MONOLITHIC within 10%
    of Fig. 2's objective.
P10 with b = (1, 3, 9, 6), >= 95% of random trials on 50,000-input
    streams are miss-free at every tested (D, tau0); here 10 seeds x 50,000 inputs at
    three grid points of the paper-faithful random-gain BLAST model (L208–L210, Table 1).
"""
import math

import pytest

from plgen import configs as C
from oracle import des, solver as SV

T1, G1, B1, V1 = C.TABLE1_T, C.TABLE1_G, C.PAPER_B, C.TABLE1_V


def _int_waits(tau, D):
    Pc, _ = SV.fig1_continuous(T1, G1, B1, V1, tau, D)
    P = [math.floor(x) for x in Pc]
    assert SV.fig1_feasible(T1, G1, B1, V1, tau, D, P)
    return [P[i] - T1[i] for i in range(4)], P


@pytest.mark.parametrize("tau,D", [(10, 50_000), (20, 100_000), (100, 350_000)])
def test_p10_miss_free_fraction(tau, D):
    w, P = _int_waits(tau, D)
    ok = 0
    seeds = range(10)
    for s in seeds:
        cfg = C.gain_model_blast(interarrival=tau, deadline=D, wait_time=tuple(w), seed=s,
                                 n_roots=50_000)
        r = des.run(cfg)
        ok += r.misses(D) == 0
        # P9: FIXED_WAIT's simulated active fraction is the Fig. 1 objective up to ceilings
        assert abs(r.active_fraction(C.FIXED_WAIT) - SV.fig1_objective(T1, P)) < 0.01
    assert ok >= 0.95 * len(seeds)


@pytest.mark.parametrize("tau,D", [(20, 25_000), (100, 25_000), (50, 100_000)])
def test_p9_monolithic_sim_vs_optimiser(tau, D):
    M, obj = SV.fig2_exhaustive(T1, G1, V1, tau, D)
    cfg = C.gain_model_blast(interarrival=tau, deadline=D, policy=C.MONOLITHIC, block_size=M,
                             seed=1, n_roots=50_000)
    r = des.run(cfg)
    assert abs(r.active_fraction(C.MONOLITHIC) / obj - 1) < 0.10
