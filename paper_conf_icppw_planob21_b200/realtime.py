"""Real-time (physical %globaltimer) operation: gains, service-time budgets, rate search.

The paper's method needs per-node service times t_i and average gains g_i
(§2.1, §2.2, Table 1) and calibrates its queue multipliers b_i
empirically (§6.2).  On B200 the t_i are not the paper's GTX-2080
cycles: they are *budgets* measured here, and the physical executor replays the
logical schedule against them.  All runs go through
the C-ABI (pipeline.Pipeline); nothing here computes the method itself.
"""
from __future__ import annotations

import math

from .pipeline import Pipeline, solve_enforced_waits, solve_monolithic

PHYS = 1  # PL_CLOCK_GLOBALTIMER


def _run(cfg, db_dev, n_bases, wl, flags=0, stream=None, over=None):
    pl = Pipeline(cfg, wl, flags=flags, stream=stream, **(over or {}))
    pl.bind_device(db_dev, n_bases)
    pl.drain()
    st = pl.stats()
    pl.close()
    return st


def measure_gains(cfg, wl, db_dev, stream=None, over=None):
    """Average gains g_i = produced_i / consumed_i from one logical-clock run."""
    st = _run(cfg.replace(clock=0, gain=None), db_dev, wl.db_len, wl, stream=stream, over=over)
    N = cfg.n_stages
    return tuple(st["produced"][i] / max(1, st["consumed"][i]) for i in range(N - 1))


def calibrate_budgets(cfg, wl, db_dev, margin=1.25, slack_ns=256, probe_t=20_000, probe_tau=100, stream=None,
                      over=None):
    """Service-time budgets t_i (ns): the longest measured firing of each node in a
    physical run with generous budgets, times `margin`, plus `slack_ns`.  The probe's
    arrivals (probe_t / probe_tau > v per period) keep node 0's vectors full."""
    N = cfg.n_stages
    probe = cfg.replace(clock=PHYS, service_time=(probe_t,) * N, wait_time=(0,) * N, interarrival=probe_tau,
                        deadline=10**12, policy=0, gain=None, ns_per_unit=1.0)
    st = _run(probe, db_dev, wl.db_len, wl, stream=stream, over=over)
    return tuple(int(math.ceil(margin * st["max_fire_ns"][i])) + slack_ns for i in range(N)), st


def solve_at(cfg, tau):
    """Fig. 1 at inter-arrival tau (None if infeasible)."""
    try:
        w, th, T, Tc = solve_enforced_waits(cfg.replace(interarrival=int(tau)))
        return w, th, T
    except RuntimeError:
        return None


def min_feasible_tau(cfg, lo=1, hi=1 << 20):
    """Smallest integer tau0 for which Fig. 1 is feasible (feasibility is monotone in tau0)."""
    if solve_at(cfg, hi) is None:
        return None
    while lo < hi:
        mid = (lo + hi) // 2
        if solve_at(cfg, mid) is None:
            lo = mid + 1
        else:
            hi = mid
    return lo


def find_rate(cfg, wl, db_dev, tries=12, grow=1.15, stream=None, log=None, over=None):
    """Smallest tau0 (ns) at which a physical FIXED_WAIT run has zero deadline misses and
    no queue overflow (budget overruns are counted and reported, not fatal: they delay
    firings, and any delay that matters shows up as a miss).  Starts at the smallest tau0
    for which Fig. 1 is feasible, grows by `grow` until a run is clean, then bisects between
    the last failing and the first clean tau0.  Returns (tau0, w, theta, T, stats)."""
    from ._pl import PlError

    def trial(tau):
        sol = solve_at(cfg, tau)
        if sol is None:
            return None
        w, th, T = sol
        c = cfg.replace(interarrival=int(tau), wait_time=tuple(w), clock=PHYS)
        try:
            st = _run(c, db_dev, wl.db_len, wl, flags=1, stream=stream, over=over)
            ok = st["misses"] == 0 and st["errors"] == 0
        except PlError:          # device-side overflow reported by drain
            st, ok = {"misses": -1, "errors": -1, "overruns": [], "max_latency_ns": -1}, False
        if log:
            log(dict(tau=tau, w=w, T=T, misses=st["misses"], overruns=st["overruns"], errors=st["errors"],
                     max_latency_ns=st["max_latency_ns"]))
        return (int(tau), w, th, T, st) if ok else None

    tau = min_feasible_tau(cfg)
    if tau is None:
        raise RuntimeError("Fig. 1 infeasible for every tau0 at this deadline")
    bad = tau - 1
    good = None
    for _ in range(tries):
        good = trial(tau)
        if good:
            break
        bad = tau
        tau = int(math.ceil(tau * grow)) + 1
    if not good:
        raise RuntimeError("no miss-free rate found")
    hi = good[0]
    while hi - bad > 1 and (hi - bad) > 0.02 * hi:
        mid = (bad + hi) // 2
        r = trial(mid)
        if r:
            good, hi = r, mid
        else:
            bad = mid
    return good


def monolithic_at(cfg, tau):
    try:
        return solve_monolithic(cfg.replace(interarrival=int(tau)))
    except RuntimeError:
        return None
