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


def _run(cfg, db_dev, n_bases, wl, flags=0, stream=None, over=None, inject=None):
    pl = Pipeline(cfg, wl, flags=flags, stream=stream, **(over or {}))
    pl.bind_device(db_dev, n_bases)
    if inject:   # (period_ns, len_ns): pl_pipeline_inject_stalls
        pl.inject_stalls(*inject)
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
                      over=None, flags=0, reps=2):
    """Service-time budgets t_i (ns): the longest measured firing of each node in a
    physical run with generous budgets, times `margin`, plus `slack_ns`.  The probe's
    arrivals (probe_t / probe_tau > v per period) keep node 0's vectors full.  `flags`
    must match the runs the budgets are for: per-item records (PL_REC_*) select the
    recording kernel, whose firings are longer.  The probe runs `reps` times and each node
    keeps the smallest of its per-run maxima: a one-off outlier (a cold first launch, a
    platform stall inside a firing) does not set a budget."""
    N = cfg.n_stages
    probe = cfg.replace(clock=PHYS, service_time=(probe_t,) * N, wait_time=(0,) * N, interarrival=probe_tau,
                        deadline=10**12, policy=0, gain=None, ns_per_unit=1.0)
    runs = [_run(probe, db_dev, wl.db_len, wl, flags=flags, stream=stream, over=over) for _ in range(max(1, reps))]
    st = dict(runs[-1], max_fire_ns=[min(r["max_fire_ns"][i] for r in runs) for i in range(N)],
              max_fire_ns_runs=[r["max_fire_ns"] for r in runs])
    return tuple(int(math.ceil(margin * st["max_fire_ns"][i])) + slack_ns for i in range(N)), st


def refine_budgets(cfg, wl, db_dev, budgets, margin=1.10, slack_ns=128, rounds=2, reps=3, flags=0, stream=None,
                   over=None, log=None, policy=0, max_lateness_ns=5000, solve_deadline=None, guard_extra=0,
                   stall_ns=100_000, lower=True):
    """Budgets re-measured at the operating point.  The probe of calibrate_budgets fires every
    node with a full vector at a period of its own; at the operating point a node can fire
    back to back (THRESHOLD_SLACK in a burst), and then its real per-firing cost is the whole
    loop -- the firing, its publish and the next decision (pl_stats.max_loop_ns) -- not the
    firing alone.  Each round finds the miss-free rate for the current budgets (find_rate),
    runs that schedule `reps` times with the kernel the budgets are for (`flags`) and sets
    t_i = ceil(margin * max(longest firing, longest loop)) + slack_ns, raising it -- and lowering
    it too unless lower=False.
    A per-run maximum above max(stall_ns, 10 t_i) is a platform stall inside a firing
    (profiles/r02_pause_control.txt), not the work: that run's value is ignored for the node.
    Stops when no budget moves by more than 2 %.  Returns (budgets, history)."""
    hist = []
    for _ in range(rounds):
        c = cfg.replace(service_time=tuple(budgets))
        if policy == 1:   # THRESHOLD_SLACK: the slack guard follows the budgets
            c = c.replace(slack_guard=int(max(budgets)) + guard_extra)
        tau, w, th, T, st = find_rate(c, wl, db_dev, stream=stream, over=over, policy=policy, flags=flags,
                                      max_lateness_ns=max_lateness_ns, solve_deadline=solve_deadline,
                                      grow=1.5)
        worst = [0] * cfg.n_stages
        for _ in range(reps):
            for _attempt in range(3):   # a run that met a platform stall measures the stall: repeat it
                s2 = _run(c.replace(interarrival=tau, wait_time=tuple(w), wait_threshold=tuple(th), clock=PHYS,
                                    policy=policy), db_dev, wl.db_len, wl, flags=flags, stream=stream, over=over)
                if not stalled(s2):
                    break
            if stalled(s2):
                continue
            for i in range(cfg.n_stages):
                x = max(s2["max_fire_ns"][i], s2["max_loop_ns"][i])
                if x <= max(stall_ns, 10 * budgets[i]):
                    worst[i] = max(worst[i], x)
        nb = tuple(int(math.ceil(margin * x)) + slack_ns if x else b for b, x in zip(budgets, worst))
        if not lower:    # keep the probe's budgets as a floor (e.g. measured at a 1/N share, L69)
            nb = tuple(max(x, y) for x, y in zip(nb, budgets))
        hist.append(dict(budgets=tuple(budgets), tau=tau, max_fire_or_loop_ns=worst, next=nb))
        if log:
            log(hist[-1])
        moved = any(abs(x - y) > 0.02 * y for x, y in zip(nb, budgets))
        budgets = nb
        if not moved:
            break
    return tuple(budgets), hist


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


STALL_NS = 1_000_000   # every node at least this late in one run: a platform SM stall (R-STALL)


def stalled(st) -> bool:
    """Whether a physical run met a platform stall: the B200 stops every SM for ~1.6 ms every
    few seconds (profiles/r02_pause_control.txt), so every node of the stream falls ~1.6 ms
    behind its schedule at once; an overloaded node alone does not look like that."""
    lat = st.get("max_lateness_ns") or [0]
    return min(lat) >= STALL_NS


def find_rate(cfg, wl, db_dev, tries=12, grow=1.15, stream=None, log=None, over=None, policy=0,
              max_lateness_ns=5000, flags=0, solve_deadline=None, max_outliers=None, start=None,
              stall_retries=2, inject=None, max_latency_ns=None):
    """Smallest tau0 (ns) at which a physical run (FIXED_WAIT, or THRESHOLD_SLACK with the
    Fig. 1-derived thresholds when policy=1) has zero deadline misses, no queue overflow
    and, unless max_lateness_ns is None, every firing starting within max_lateness_ns of its
    scheduled time.  The lateness bound is the sustainability check: a node whose real
    per-firing cycle (firing + publish + next decision, pl_stats.max_loop_ns) exceeds its
    period falls further behind with every firing, which a finite stream can hide inside D
    (budget overruns are counted and reported, not fatal).  Starts at the smallest tau0
    for which Fig. 1 is feasible, grows by `grow` until a run is clean, then bisects between
    the last failing and the first clean tau0.  The trial runs use the kernel selected by
    `flags` (default: the record-free kernel that the bench times; misses are counted on the
    device either way).  `solve_deadline`: the deadline Fig. 1 is solved at (default cfg's D; a
    platform-stall allowance is kept out of it, DESIGN.md R-STALL), while misses count against
    cfg's D.  `start`: the first tau0 tried (default: the smallest Fig. 1-feasible one).  A
    failing run that met a platform stall (stalled()) is repeated up to `stall_retries` times: it
    says nothing about the rate.  `inject` = (period_ns, len_ns): every trial run carries injected
    platform-length stalls (pl_pipeline_inject_stalls), and the criterion becomes zero misses
    ACROSS them -- the pipeline must catch up after each within D (R-STALL); the 5 % outlier
    bound then cannot apply (a stalled item is late by construction) and is not checked.
    `max_latency_ns`: a run also needs its largest measured latency within this bound (a margin
    under D: near the edge the worst latency across stalls is not monotone in tau0, and a run that
    just clears D says little about the next one).  
    Returns (tau0, w, theta, T, stats)."""
    from ._pl import PlError
    scfg = cfg if solve_deadline is None else cfg.replace(deadline=int(solve_deadline))

    def trial(tau):
        sol = solve_at(scfg, tau)
        if sol is None:
            return None
        w, th, T = sol
        c = cfg.replace(interarrival=int(tau), wait_time=tuple(w), wait_threshold=tuple(th), clock=PHYS,
                        policy=policy)
        for attempt in range(stall_retries + 1):
            try:
                st = _run(c, db_dev, wl.db_len, wl, flags=flags, stream=stream, over=over, inject=inject)
                ok = (st["misses"] == 0 and st["miss_events"] == 0 and st["miss_events_ns"] == 0
                      and st["errors"] == 0)
                if max_lateness_ns is not None:
                    ok = ok and max(st["max_lateness_ns"]) <= max_lateness_ns
                if max_latency_ns is not None:
                    ok = ok and st["max_latency_ns"] <= max_latency_ns
                if max_outliers is not None and not inject:   # north_star 5 % per-item agreement (R-AGREE)
                    ok = ok and st["latency_outliers"] <= max_outliers
            except PlError:          # device-side overflow reported by drain
                st, ok = {"misses": -1, "miss_events_ns": -1, "errors": -1, "overruns": [], "max_latency_ns": -1,
                          "max_lateness_ns": []}, False
            if ok or inject or not stalled(st):
                break
        if log:
            log(dict(tau=tau, w=w, T=T, misses=st["misses"], overruns=st["overruns"], errors=st["errors"],
                     max_latency_ns=st["max_latency_ns"], max_lateness_ns=st["max_lateness_ns"],
                     outliers=st.get("latency_outliers")))
        return (int(tau), w, th, T, st) if ok else None

    tau = min_feasible_tau(scfg)
    if tau is None:
        raise RuntimeError("Fig. 1 infeasible for every tau0 at this deadline")
    if start is not None and start > tau:
        tau = int(start)
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


def calibrate_b(cfg, wl=None, db_dev=None, target=0.95, quantile=0.95, max_iter=10, log=None, stream=None,
                arrivals=None, over=None):
    """The paper's empirical b calibration, run on the device.

    Start from b = 1 ("optimistic ... worst-case closely matches the average"), solve Fig. 1,
    run all cfg.n_streams streams (independent seeds) in one launch, and accept once at least
    `target` of them are miss-free.  Otherwise raise b_i to the `quantile` of the streams'
    measured input-queue peaks divided by v -- L133 defines b_i v as the queue's maximum size
    -- (or by one if that would not change b), re-solve and repeat.
    Returns dict(b, w, T, miss_free, iterations, history)."""
    import numpy as np
    N, v = cfg.n_stages, cfg.vector_width
    b = [1] * N
    hist = []
    for it in range(max_iter):
        c = cfg.replace(b=tuple(b))
        try:
            w, th, T, Tc = solve_enforced_waits(c)
        except RuntimeError:
            return dict(b=tuple(b), w=None, T=None, miss_free=0.0, iterations=it, history=hist, infeasible=True)
        c = c.replace(wait_time=tuple(w))
        pl = Pipeline(c, wl, flags=1, stream=stream, arrivals=arrivals, **(over or {}))
        if wl is not None:
            pl.bind_device(db_dev, wl.db_len)
        else:
            pl.push(None, c.n_roots)
        pl.drain()
        lat, lat_ns = pl.latency()
        peaks = pl.queue_peaks()
        pl.close()
        L = lat_ns if c.clock == PHYS else lat
        limit = c.deadline * (c.ns_per_unit if c.clock == PHYS else 1)
        per = L[: (len(L) // c.n_streams) * c.n_streams].reshape(c.n_streams, -1)
        mf = float(((per > limit).sum(axis=1) == 0).mean())
        qb = [int(math.ceil(x / v)) for x in np.quantile(peaks, quantile, axis=0)]
        rec = dict(iteration=it, b=tuple(b), T=T, miss_free=mf, queue_peak_q=[int(x) for x in
                   np.quantile(peaks, quantile, axis=0)], b_from_queues=qb)
        hist.append(rec)
        if log:
            log(rec)
        if mf >= target:
            return dict(b=tuple(b), w=tuple(w), T=T, miss_free=mf, iterations=it + 1, history=hist)
        nb = [max(b[i], qb[i]) for i in range(N)]
        if nb == b:   # queues already within b_i v: raise the node whose queue is closest to its bound
            ratio = [peaks[:, i].max() / (b[i] * v) for i in range(N)]
            nb[int(np.argmax(ratio))] += 1
        b = nb
    return dict(b=tuple(b), w=None, T=None, miss_free=hist[-1]["miss_free"], iterations=max_iter, history=hist)
