"""Pins for oracle.solver.

Fig. 1 is pinned by two closed forms that follow from the
mathematics (Cauchy–Schwarz when only the deadline binds; the stability chain
when only L125/L131 bind), by integer brute force on small boxes, and by the
paper's qualitative statements about Figs. 3/4 (L236–L255).  Fig. 2 (L165–L180)
is pinned by a hand-worked example.
"""
import math

import pytest

from plgen import configs as C
from oracle import solver as SV

T1, G1, B1, V1 = C.TABLE1_T, C.TABLE1_G, C.PAPER_B, C.TABLE1_V


def test_fig1_deadline_closed_form_table1():
    """Only the deadline binds (tau0 large, D moderate): Lagrange/Cauchy–Schwarz gives
    P_i = D sqrt(t_i/b_i) / sum_j sqrt(t_j b_j) and T* = (sum sqrt(t_i b_i))^2 / (N D)."""
    D, tau = 100_000, 100
    s = sum(math.sqrt(t * b) for t, b in zip(T1, B1))
    P = [D * math.sqrt(t / b) / s for t, b in zip(T1, B1)]
    # preconditions: the other constraints are slack at this P
    assert all(P[i] > T1[i] for i in range(4)) and P[0] < V1 * tau
    assert all(G1[i - 1] * P[i] < P[i - 1] for i in range(1, 4))
    Tstar = s * s / (4 * D)
    assert abs(Tstar * D - 16788) < 1.0            # = 16,788 / D
    Pc, Tc = SV.fig1_continuous(T1, G1, B1, V1, tau, D)
    assert abs(Tc - Tstar) < 1e-6 * Tstar
    for a, b in zip(Pc, P):
        assert abs(a - b) < 1e-3 * b


def test_fig1_stability_closed_form_table1():
    """Deadline slack (D huge): P_0 = v tau0, P_i = P_{i-1}/g_{i-1}, T = (1/N) sum t_i G_i/(v tau0)."""
    tau, D = 10, 10**9
    P = [V1 * tau]
    for i in range(1, 4):
        P.append(P[-1] / G1[i - 1])
    assert all(P[i] >= T1[i] for i in range(4))
    G = SV.gains_G(G1, 4)
    T = sum(T1[i] * G[i] for i in range(4)) / (4 * V1 * tau)
    assert abs(T * tau - 1.969) < 1e-3              # = 1.969 / tau0
    Pc, Tc = SV.fig1_continuous(T1, G1, B1, V1, tau, D)
    assert abs(Tc - T) < 1e-6 * T


@pytest.mark.parametrize("prob", [
    ((64, 96), (0.5,), (1, 2), 32, 4, 500),
    ((5, 9, 4), (0.7, 1.6), (1, 2, 3), 4, 3, 120),
    ((3, 7), (0.4,), (2, 1), 2, 5, 60),
    ((6, 4, 5), (0.5, 0.9), (1, 1, 1), 8, 2, 90),
])
def test_fig1_integer_bruteforce_vs_continuous(prob):
    t, g, b, v, tau, D = prob
    Pi, Ti = SV.fig1_bruteforce_int(t, g, b, v, tau, D)
    Pc, Tc = SV.fig1_continuous(t, g, b, v, tau, D)
    assert Pi is not None and Pc is not None
    assert SV.fig1_feasible(t, g, b, v, tau, D, Pi)
    assert Ti >= Tc - 1e-9
    # rounding cost is bounded by the objective's sensitivity to one unit per coordinate
    assert Ti - Tc <= sum(t[i] / (Pc[i] - 1) - t[i] / Pc[i] for i in range(len(t))) / len(t) * 4 + 1e-9


def test_fig1_c1_worked_example():
    """config 1, D = 500 -> (P0, P1) = (128, 186), T = 0.5081."""
    Pi, Ti = SV.fig1_bruteforce_int((64, 96), (0.5,), (1, 2), 32, 4, 500)
    assert Pi == [128, 186]
    assert abs(Ti - 0.5 * (64 / 128 + 96 / 186)) < 1e-15


def test_fig1_infeasible_below_sum_bt():
    """sum_i b_i t_i = 23,288 > 2e4: no w >= 0 meets L135 at D = 2e4."""
    assert sum(t * b for t, b in zip(T1, B1)) == 23288
    assert SV.fig1_continuous(T1, G1, B1, V1, 50, 20_000) == (None, None)


def test_fig2_hand_example_c1():
    """c1, D = 500, b = S = 1: Tbar(M) = ceil(M/32) 64 + ceil(M/64) 96.
    M = 64: Tbar = 2*64 + 1*96 = 224 <= 256 = M tau0 and 256 + 224 = 480 <= 500; objective 0.875.
    M > 64: Tbar(65) = 3*64 + 2*96 = 384 -> 260 + 384 > 500 (and larger M only worse).
    M < 64 stable only for 56 <= M <= 64 (Tbar = 224), objective 224/(4M) >= 0.875."""
    M, obj = SV.fig2_exhaustive((64, 96), (0.5,), 32, 4, 500)
    assert (M, obj) == (64, 0.875)
    assert SV.tbar(64, (64, 96), (0.5,), 32) == 224


def test_fig2_infeasible_fast_arrivals():
    """At tau0 <= 5 the monolithic pipeline cannot keep up: Tbar(M)/M -> sum G_i t_i / v = 7.875 > tau0."""
    G = SV.gains_G(G1, 4)
    assert abs(sum(G[i] * T1[i] for i in range(4)) / V1 - 7.875) < 1e-3
    assert SV.fig2_exhaustive(T1, G1, V1, 5, 350_000) == (None, None)


def test_thresholds_formula_examples():
    # theta_i = clamp(floor(G_i P_i / tau0), 1, v): c1, P = (128, 186), tau0 = 4
    assert SV.thresholds((0.5,), (128, 186), 4, 32) == [32, 23]
    assert SV.thresholds((0.5,), (2, 3), 4, 32) == [1, 1]


def _enf(tau, D):
    r = SV.fig1_continuous(T1, G1, B1, V1, tau, D)
    return r[1]


def _mono(tau, D):
    return SV.fig2_exhaustive(T1, G1, V1, tau, D)[1]


def test_paper_fig4_claims():
    """enforced waits beat monolithic by >= 0.4 absolute at the fastest
    arrival rates with deadline slack; monolithic dominates by a similar amount for slow
    arrivals and little deadline slack."""
    assert _mono(10, 350_000) - _enf(10, 350_000) >= 0.4
    assert _mono(10, 100_000) - _enf(10, 100_000) >= 0.4
    assert _enf(100, 25_000) - _mono(100, 25_000) >= 0.4


def test_paper_fig3_sensitivities():
    """enforced ~ 1/D and insensitive to tau0 except at the smallest
    values; monolithic mostly insensitive to D and ~ 1/tau0."""
    e1, e2 = _enf(50, 50_000), _enf(50, 100_000)
    assert abs(e1 / e2 - 2.0) < 0.05                      # ~ 1/D (deadline-bound regime)
    assert abs(_enf(20, 100_000) - _enf(100, 100_000)) < 0.02
    m1, m2 = _mono(20, 100_000), _mono(20, 350_000)
    assert abs(m1 - m2) < 0.05                            # insensitive to D
    assert abs(_mono(50, 350_000) * 50 / (_mono(100, 350_000) * 100) - 1) < 0.1   # ~ 1/tau0
