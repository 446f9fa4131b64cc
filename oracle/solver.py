"""The paper's two optimisation problems, by their definitions (ORACLE — test infrastructure).

Fig. 1, enforced waiting:
    min T(w) = (1/N) sum_i t_i / (t_i + w_i)
    s.t. (t_0 + w_0) rho_0 <= v                      (L125/L145; reading A3)
         (t_i + w_i) g_{i-1} <= t_{i-1} + w_{i-1}    (L131/L147)
         sum_i b_i (t_i + w_i) <= D                   (L135/L149)
         w_i >= 0                                     (L140)
Fig. 2, monolithic:
    min rho_0 Tbar(M) / M  s.t. Tbar(M) <= M/rho_0,  b M/rho_0 + S Tbar(M) <= D,
    Tbar(M) = sum_i ceil(M G_i / v) t_i               (L176, L188)

Integer wait times (reading A17): the oracle's integer optimum is the plain
enumeration of every integer P = t + w in the feasible box (small problems
only).  The continuous Fig. 1 optimum uses scipy SLSQP (a library primitive)
from several starts.  Fig. 2 is solved by enumerating M (its definition).

Floating-point decisions that yield integers (ceil in Tbar, floor in theta)
are taken in IEEE double, with G_i accumulated left to right (DESIGN.md R-FP).
"""
from __future__ import annotations

import itertools
import math


def gains_G(g, N):
    G = [1.0]
    for i in range(N - 1):
        G.append(G[-1] * g[i])
    return G


def fig1_objective(t, P):
    return sum(t[i] / P[i] for i in range(len(t))) / len(t)


def fig1_feasible(t, g, b, v, tau, D, P, eps=0.0):
    N = len(t)
    if any(P[i] < t[i] - eps for i in range(N)):
        return False
    if P[0] > v * tau + eps:                       # (t0+w0) rho0 <= v  <=>  P0 <= v tau0
        return False
    for i in range(1, N):
        if P[i] * g[i - 1] > P[i - 1] + eps:
            return False
    return sum(b[i] * P[i] for i in range(N)) <= D + eps


def fig1_bruteforce_int(t, g, b, v, tau, D):
    """Every integer P with t_i <= P_i and the constraints; min T, ties -> lexicographically
    smallest w.  Exponential: tiny problems only.  Returns (P, T) or (None, None)."""
    N = len(t)
    ub = [min(v * tau, D)] + [D] * (N - 1)
    ub = [min(ub[i], (D - sum(b[j] * t[j] for j in range(N) if j != i)) // b[i]) for i in range(N)]
    best = None
    for P in itertools.product(*[range(t[i], ub[i] + 1) for i in range(N)]):
        if not fig1_feasible(t, g, b, v, tau, D, P):
            continue
        T = fig1_objective(t, P)
        key = (T, tuple(P[i] - t[i] for i in range(N)))
        if best is None or key < best[0]:
            best = (key, P)
    if best is None:
        return None, None
    return list(best[1]), best[0][0]


def fig1_exact_int_absorb(t, g, b, v, tau, D):
    """Exact integer Fig. 1 optimum for N = 2 or 3 at moderate sizes.  For fixed P_1..P_{N-1}
    the objective falls as P_0 grows, and P_0 is constrained only by
    max(t_0, g_0 P_1) <= P_0 <= min(v tau0, (D - sum_{j>=1} b_j P_j) / b_0), so the best P_0 is
    the top of that interval: enumerating every integer P_1..P_{N-1} (numpy grid) with that
    P_0 is an exhaustive search.  Returns the optimal objective (or None if infeasible)."""
    import numpy as np
    N = len(t)
    assert N in (2, 3)
    ub = [(D - sum(b[j] * t[j] for j in range(N) if j != i)) // b[i] for i in range(N)]
    axes = [np.arange(t[i], ub[i] + 1, dtype=np.int64) for i in range(1, N)]
    if any(len(a) == 0 for a in axes):
        return None
    grid = np.meshgrid(*axes, indexing="ij")
    P = [None] + [x.ravel() for x in grid]
    rest = sum(b[j] * P[j] for j in range(1, N))
    P0 = np.minimum((D - rest) // b[0], int(math.floor(v * tau)))
    ok = (P0 >= t[0]) & (P[1] * g[0] <= P0)
    if N == 3:
        ok &= P[2] * g[1] <= P[1]
    if not ok.any():
        return None
    T = t[0] / P0[ok].astype(float)
    for j in range(1, N):
        T = T + t[j] / P[j][ok].astype(float)
    return float(T.min()) / N


def fig1_continuous(t, g, b, v, tau, D, starts=8, seed=0):
    """Continuous Fig. 1 optimum by scipy SLSQP from several feasible-ish starts."""
    import numpy as np
    from scipy.optimize import minimize
    N = len(t)
    t = np.asarray(t, float)
    b = np.asarray(b, float)
    cons = [{"type": "ineq", "fun": lambda P: v * tau - P[0]},
            {"type": "ineq", "fun": lambda P: D - float(np.dot(b, P))}]
    for i in range(1, N):
        cons.append({"type": "ineq", "fun": lambda P, i=i: P[i - 1] - g[i - 1] * P[i]})
    bounds = [(t[i], None) for i in range(N)]
    rng = np.random.default_rng(seed)
    best = None
    for s in range(starts):
        x0 = t * (1.0 + rng.random(N) * (1.0 if s else 0.0))
        r = minimize(lambda P: float(np.sum(t / P)) / N, x0, method="SLSQP", bounds=bounds,
                     constraints=cons, options={"ftol": 1e-14, "maxiter": 2000})
        if not r.success:
            continue
        P = r.x
        if not fig1_feasible(list(t), g, list(b), v, tau, D, list(P), eps=1e-6 * D):
            continue
        if best is None or r.fun < best[1]:
            best = (list(P), float(r.fun))
    return best if best else (None, None)


def thresholds(g, P, tau, v):
    """theta_i = clamp(floor(G_i P_i / tau0), 1, v)  (reading R-THETA)."""
    G = gains_G(g, len(P))
    return [max(1, min(v, math.floor(G[i] * P[i] / tau))) for i in range(len(P))]


def tbar(M, t, g, v):
    """Tbar(M) = sum_i ceil(M G_i / v) t_i."""
    G = gains_G(g, len(t))
    return sum(math.ceil(M * G[i] / v) * t[i] for i in range(len(t)))


def fig2_exhaustive(t, g, v, tau, D, b=1, S=1.0):
    """Enumerate M = 1, 2, ... while b M tau0 + S Tbar(M) <= D (LHS non-decreasing in M);
    keep the M minimising Tbar(M)/(M tau0) among those with Tbar(M) <= M tau0.
    Ties -> smallest M.  Returns (M, objective) or (None, None)."""
    best = None
    M = 1
    while b * M * tau + S * tbar(M, t, g, v) <= D:
        tb = tbar(M, t, g, v)
        if tb <= M * tau:
            obj = tb / (M * tau)
            if best is None or obj < best[1]:
                best = (M, obj)
        M += 1
    return best if best else (None, None)
