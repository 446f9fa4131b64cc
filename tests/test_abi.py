"""Host-side checks of the C-ABI library (no GPU needed): it loads, exports every
symbol include/pl.h declares, validates configurations, and its host solvers agree
with the oracle's definitions of Fig. 1 / Fig. 2."""
import ctypes
import os
import re

import pytest

from plgen import configs as C
from oracle import solver as SV

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "pl.h")).read()
    return sorted(set(re.findall(r"\b(pl_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    from paper_conf_icppw_planob21_b200 import _pl
    lib = ctypes.CDLL(_pl.LIB_PATH)
    names = _declared()
    assert "pl_pipeline_create" in names and len(names) >= 18
    for n in names:
        assert hasattr(lib, n), n
    assert set(_pl.EXPORTED) == set(names)


def test_struct_sizes_match_header():
    """ctypes mirrors of the public structs have the C sizes (checked against offsets)."""
    from paper_conf_icppw_planob21_b200 import _pl
    assert ctypes.sizeof(_pl.pl_match) == 24
    assert ctypes.sizeof(_pl.pl_firing) == 32
    assert ctypes.sizeof(_pl.pl_stage) == 32


def test_create_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_icppw_planob21_b200 import Pipeline, PlError
    with pytest.raises(PlError) as ei:
        Pipeline(C.c1(wait_time=(64, 90)))
    assert "PL_EDEVICE" in str(ei.value)


@pytest.mark.parametrize("bad", [dict(vector_width=48), dict(interarrival=0), dict(deadline=0),
                                 dict(service_time=(0, 96)), dict(wait_time=(-1, 0))])
def test_validation_errors(bad):
    from paper_conf_icppw_planob21_b200 import Pipeline, PlError
    cfg = C.c1(wait_time=(64, 90)).replace(**bad)
    with pytest.raises(PlError) as ei:
        Pipeline(cfg)
    assert "PL_EINVAL" in str(ei.value)


@pytest.mark.parametrize("prob", [
    ((64, 96), (0.5,), (1, 2), 32, 4, 500),
    ((5, 9, 4), (0.7, 1.6), (1, 2, 3), 4, 3, 120),
    ((3, 7), (0.4,), (2, 1), 2, 5, 60),
    ((6, 4, 5), (0.5, 0.9), (1, 1, 1), 8, 2, 90),
    ((7, 3, 9), (1.5, 0.3), (2, 1, 1), 4, 5, 110),
])
def test_solver_fig1_matches_oracle_bruteforce(prob):
    from paper_conf_icppw_planob21_b200 import solve_enforced_waits
    t, g, b, v, tau, D = prob
    stages = [C.Stage(C.BERNOULLI, 0.5, 1)] * len(t)
    cfg = C.Config(name="s", stages=stages, service_time=t, vector_width=32, deadline=D,
                   interarrival=tau, b=b, gain=g)
    cfg.vector_width = v            # solver accepts any v (the executor restricts it)
    Pi, Ti = SV.fig1_bruteforce_int(t, g, b, v, tau, D)
    w, th, T, Tc = solve_enforced_waits(cfg)
    assert [w[i] + t[i] for i in range(len(t))] == Pi
    assert abs(T - Ti) < 1e-15
    Pc, Tco = SV.fig1_continuous(t, g, b, v, tau, D)
    assert abs(Tc - Tco) < 1e-7 * Tco
    assert th == SV.thresholds(g, Pi, tau, v)


@pytest.mark.parametrize("tau,D", [(3, 25_000), (5, 50_000), (10, 50_000), (10, 350_000), (20, 100_000),
                                   (50, 200_000), (100, 25_000), (100, 350_000)])
def test_solver_fig1_table1_grid(tau, D):
    from paper_conf_icppw_planob21_b200 import solve_enforced_waits
    cfg = C.gain_model_blast(interarrival=tau, deadline=D)
    w, th, T, Tc = solve_enforced_waits(cfg)
    Pc, Tco = SV.fig1_continuous(C.TABLE1_T, C.TABLE1_G, C.PAPER_B, 128, tau, D)
    assert abs(Tc - Tco) < 1e-7 * Tco
    P = [w[i] + C.TABLE1_T[i] for i in range(4)]
    assert SV.fig1_feasible(C.TABLE1_T, C.TABLE1_G, C.PAPER_B, 128, tau, D, P)
    assert Tco - 1e-12 <= T <= Tco * (1 + 2e-3)


@pytest.mark.parametrize("tau,D", [(1, 350_000), (2, 50_000), (50, 20_000)])
def test_solver_fig1_infeasible(tau, D):
    from paper_conf_icppw_planob21_b200 import PlError, solve_enforced_waits
    if D == 20_000 or tau <= 2:
        with pytest.raises(PlError) as ei:
            solve_enforced_waits(C.gain_model_blast(interarrival=tau, deadline=D))
        assert "PL_EINFEASIBLE" in str(ei.value)


@pytest.mark.parametrize("tau,D", [(10, 25_000), (10, 350_000), (20, 20_000), (50, 100_000), (100, 25_000)])
def test_solver_fig2_matches_oracle(tau, D):
    from paper_conf_icppw_planob21_b200 import solve_monolithic
    M, T = solve_monolithic(C.gain_model_blast(interarrival=tau, deadline=D))
    Mo, To = SV.fig2_exhaustive(C.TABLE1_T, C.TABLE1_G, 128, tau, D)
    assert (M, T) == (Mo, To)


def _random_fig1_problem(rnd):
    N = rnd.randint(1, 3)
    t = tuple(rnd.randint(1, 9) for _ in range(N))
    g = tuple(round(rnd.uniform(0.2, 2.5), 3) for _ in range(N - 1))
    b = tuple(rnd.randint(1, 3) for _ in range(N))
    v = rnd.choice([2, 4, 8])
    tau = rnd.randint(1, 6)
    D = rnd.randint(sum(x * y for x, y in zip(t, b)), 4 * sum(x * y for x, y in zip(t, b)) + 40)
    return t, g, b, v, tau, D


@pytest.mark.parametrize("seed", range(40))
def test_solver_fig1_random_vs_bruteforce(seed):
    """Property: on random small problems the C++ Fig. 1 solver returns exactly the integer
    optimum of the oracle's brute-force enumeration (or both report infeasible)."""
    import random
    from paper_conf_icppw_planob21_b200 import PlError, solve_enforced_waits
    t, g, b, v, tau, D = _random_fig1_problem(random.Random(seed))
    cfg = C.Config(name="r", stages=[C.Stage(C.BERNOULLI, 0.5, 1)] * len(t), service_time=t, vector_width=32,
                   deadline=D, interarrival=tau, b=b, gain=g)
    cfg.vector_width = v
    Pi, Ti = SV.fig1_bruteforce_int(t, g, b, v, tau, D)
    try:
        w, th, T, Tc = solve_enforced_waits(cfg)
    except PlError:
        assert Pi is None
        return
    assert Pi is not None
    assert abs(T - Ti) < 1e-12, (t, g, b, v, tau, D, [w[i] + t[i] for i in range(len(t))], Pi)


@pytest.mark.parametrize("seed", range(60))
def test_solver_fig1_random_vs_exact_absorb(seed):
    """Larger random problems (b_i up to 16, deadlines of thousands of units: the regime where
    rounding the b_i > 1 stages down frees slack for another stage) against the oracle's exact
    search (every P_1..P_{N-1}, P_0 at the top of its feasible interval)."""
    import random
    from paper_conf_icppw_planob21_b200 import PlError, solve_enforced_waits
    rnd = random.Random(1000 + seed)
    N = rnd.choice([2, 3])
    t = tuple(rnd.randint(20, 300) for _ in range(N))
    g = tuple(round(rnd.uniform(0.3, 2.0), 3) for _ in range(N - 1))
    b = tuple(rnd.randint(1, 16) for _ in range(N))
    v = rnd.choice([16, 32, 128])
    tau = rnd.randint(2, 40)
    base = sum(x * y for x, y in zip(t, b))
    D = rnd.randint(base, min(3 * base, base + 2500 * min(b)))
    cfg = C.Config(name="r", stages=[C.Stage(C.BERNOULLI, 0.5, 1)] * N, service_time=t, vector_width=32,
                   deadline=D, interarrival=tau, b=b, gain=g)
    cfg.vector_width = v
    To = SV.fig1_exact_int_absorb(t, g, b, v, tau, D)
    try:
        w, th, T, Tc = solve_enforced_waits(cfg)
    except PlError:
        assert To is None
        return
    assert To is not None
    assert abs(T - To) <= 1e-12 * To, (t, g, b, v, tau, D, [w[i] + t[i] for i in range(N)])


def test_solver_fig1_advisor_case():
    """The case the round-1 review found (t=(2124,1196,1743,2851), g=(.5,1,.5), b=(1,16,7,16),
    v=256, tau0=56, D=103030): P_0 = 8654 is feasible and better than 8653."""
    from paper_conf_icppw_planob21_b200 import solve_enforced_waits
    t, g, b, v, tau, D = (2124, 1196, 1743, 2851), (0.5, 1.0, 0.5), (1, 16, 7, 16), 256, 56, 103030
    cfg = C.Config(name="r", stages=[C.Stage(C.BERNOULLI, 0.5, 1)] * 4, service_time=t, vector_width=32,
                   deadline=D, interarrival=tau, b=b, gain=g)
    cfg.vector_width = v
    w, th, T, Tc = solve_enforced_waits(cfg)
    P = [w[i] + t[i] for i in range(4)]
    assert SV.fig1_feasible(t, g, b, v, tau, D, P)
    assert P[0] >= 8654, P
