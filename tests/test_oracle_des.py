"""Pins for oracle.des (SURVEY.md §8(c) P1–P6).

P1  FIXED_WAIT active time over [0, H) equals the exact closed form for any data
    (§4.1 L105–L119 with the ceilings kept).
P2  single-node regular streams: closed-form latencies (L63, L69, L97).
P3  THRESHOLD_SLACK utilisation on a regular fixed-gain pipeline.
P4  conservation invariants after every event (north_star).
P5  node-order permutation invariance of same-time events (reading R-ORDER).
P6  an independent time-stepped enumerator of every fire/wait schedule on tiny
    streams: the DES's schedule is one of them with identical latencies and
    active time, and the clairvoyant optimum is no worse than the policy.
"""
import itertools
import random

import pytest

from plgen import configs as C
from oracle import des


def gm_cfg(N, t, w, v, tau, X, seed=0, policy=C.FIXED_WAIT, theta=None, D=10**9):
    kinds = [C.Stage(C.BERNOULLI, 0.6, 1), C.Stage(C.POISSON_CAPPED, 1.5, 4),
             C.Stage(C.BERNOULLI, 0.5, 1), C.Stage(C.FIXED_GAIN, 2.0, 2)]
    st = kinds[:N]
    return C.Config(name="t", stages=st, service_time=tuple(t), vector_width=v, deadline=D,
                    interarrival=tau, b=(1,) * N, wait_time=tuple(w) if w else None,
                    wait_threshold=tuple(theta) if theta else None, policy=policy,
                    n_roots=X, seed=seed)


@pytest.mark.parametrize("case", range(12))
def test_p1_fixed_wait_active_closed_form(case):
    rnd = random.Random(case)
    N = rnd.randint(1, 4)
    t = [rnd.randint(3, 40) for _ in range(N)]
    w = [rnd.randint(0, 60) for _ in range(N)]
    v = rnd.choice([2, 4, 8, 32])
    tau = rnd.randint(1, 9)
    X = rnd.randint(1, 400)
    cfg = gm_cfg(N, t, w, v, tau, X, seed=case)
    r = des.run(cfg)
    s = r.streams[0]
    H = X * tau
    for i in range(N):
        P = t[i] + w[i]
        closed = (H // P) * t[i] + min(t[i], H % P)
        assert s.active_H[i] == closed, (i, s.active_H[i], closed)
    # large-X limit of L119: (1/N) sum t_i/(t_i+w_i)
    T = r.active_fraction(C.FIXED_WAIT)
    lim = sum(t[i] / (t[i] + w[i]) for i in range(N)) / N
    assert abs(T - lim) <= sum(t) / (N * H) + 1e-12


@pytest.mark.parametrize("case", range(12))
def test_p1_drain_window_closed_form(case):
    """The drain-inclusive accounting (SURVEY §8(c) C-D "Outputs"): over [0, T_end] FIXED_WAIT
    charges every slot m P_i < T_end, clipped -- floor(T_end/P) t + min(t, T_end mod P) per node
    for ANY data (L97: empty firings are charged), and THRESHOLD_SLACK charges t_i per firing
    (every firing ends by T_end, the last completion)."""
    rnd = random.Random(100 + case)
    N = rnd.randint(1, 4)
    t = [rnd.randint(3, 40) for _ in range(N)]
    w = [rnd.randint(0, 60) for _ in range(N)]
    v = rnd.choice([2, 4, 8, 32])
    tau = rnd.randint(1, 9)
    X = rnd.randint(1, 400)
    r = des.run(gm_cfg(N, t, w, v, tau, X, seed=case))
    s = r.streams[0]
    for i in range(N):
        P = t[i] + w[i]
        assert s.active_drain[i] == (s.T_end // P) * t[i] + min(t[i], s.T_end % P), i
    th = [rnd.randint(1, v) for _ in range(N)]
    r = des.run(gm_cfg(N, t, None, v, tau, X, seed=case, policy=C.THRESHOLD_SLACK, theta=th, D=10**4))
    s = r.streams[0]
    for i in range(N):
        assert s.active_drain[i] == s.n_firings[i] * t[i], i
    acc = sum(s.active_drain)
    assert r.active_fraction_drain(C.THRESHOLD_SLACK) == acc / (N * s.T_end)


@pytest.mark.parametrize("tau,P,t0,v", [(4, 128, 64, 32), (3, 10, 7, 4), (5, 5, 5, 1), (2, 9, 1, 8)])
def test_p2_fixed_wait_single_node_latency(tau, P, t0, v):
    assert P <= v * tau
    X = 97
    cfg = C.Config(name="p2", stages=[C.Stage(C.KEEP_EVERY, 1.0, 1)], service_time=(t0,),
                   vector_width=v, deadline=10**9, interarrival=tau, b=(1,), wait_time=(P - t0,),
                   n_roots=X)
    r = des.run(cfg)
    for rr in range(X):
        expect = -(-rr * tau // P) * P - rr * tau + t0       # ceil(r tau / P) P - r tau + t0
        assert r.lat[rr] == expect, (rr, r.lat[rr], expect)


@pytest.mark.parametrize("tau,t0,v,X", [(4, 64, 32, 100), (3, 5, 4, 23), (1, 8, 8, 64)])
def test_p2_threshold_single_node_latency(tau, t0, v, X):
    D = 10**6
    R0 = t0
    assert t0 <= v * tau and (v - 1) * tau < D - R0
    cfg = C.Config(name="p2t", stages=[C.Stage(C.KEEP_EVERY, 1.0, 1)], service_time=(t0,),
                   vector_width=v, deadline=D, interarrival=tau, b=(1,), wait_threshold=(v,),
                   policy=C.THRESHOLD_SLACK, n_roots=X)
    r = des.run(cfg)
    full = (X // v) * v
    for rr in range(full):
        assert r.lat[rr] == (v - 1 - rr % v) * tau + t0
    # last partial group is slack-forced at a(head) + D - R_0
    for rr in range(full, X):
        assert r.lat[rr] == full * tau + D - R0 + t0 - rr * tau


def test_p3_threshold_regular_pipeline_utilisation():
    """c1r: S0 keeps even roots (G_1 = 1/2), S1 gain 2; theta = (32, 16).  Node 0 fires every
    theta_0 arrivals, node 1 once per node-0 firing: util -> (1/N) sum rho0 G_i t_i / theta_i."""
    cfg = C.c1r(policy=C.THRESHOLD_SLACK, wait_threshold=(32, 16))
    r = des.run(cfg)
    t, tau = cfg.service_time, cfg.interarrival
    G = (1.0, 0.5)
    expect = sum(G[i] * t[i] / ((32, 16)[i] * tau) for i in range(2)) / 2
    assert abs(r.active_fraction(C.THRESHOLD_SLACK) - expect) < 5e-4
    s = r.streams[0]
    assert s.n_firings == [-(-100_000 // 32)] * 2          # ceil(X / theta_0) groups
    assert s.n_empty == [0, 0]


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_p4_conservation(policy, seed):
    cfg = gm_cfg(3, (5, 9, 4), (7, 3, 11), 4, 2, 150, seed=seed, policy=policy,
                 theta=(3, 2, 4), D=120)
    fns = des.make_stage_fns(cfg, None)
    des.simulate_stream(cfg, fns, 0, 150, check_invariants=True)


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_p5_node_order_permutation(policy):
    cfg = gm_cfg(3, (4, 6, 4), (4, 0, 2), 4, 2, 120, seed=3, policy=policy, theta=(3, 2, 2), D=80)
    fns = des.make_stage_fns(cfg, None)
    ref = des.simulate_stream(cfg, fns, 0, 120)
    for perm in itertools.permutations(range(3)):
        r = des.simulate_stream(cfg, fns, 0, 120, node_order=perm)
        assert (r.lat, r.trace, sorted(r.firings), r.active_H) == (ref.lat, ref.trace, sorted(ref.firings), ref.active_H)


# ----------------------------------------------------------------- P6 enumerator

def _enum_step_semantics(N, t, v, tau, X, fns, decide):
    """Independent time-stepped executor of the paper's model (§2):
    at each integer time T: completions, then arrivals, then `decide(T, state)` returns
    the set of idle nodes that fire now (taking min(|Q|, v) entries).  Returns
    (lat tuple, [(node, start, n)] non-empty firings).  Written separately from oracle.des."""
    Q = [[] for _ in range(N)]
    busy = [None] * N                   # (end, entries)
    lat = [-1] * X
    log = []
    qmax = [0] * N                      # longest queue at a firing decision (L133)
    T = 0
    arrived = 0
    while True:
        for i in range(N):
            if busy[i] and busy[i][0] == T:
                for e in busy[i][1]:
                    ch = fns[i](e)
                    if i < N - 1 and ch:
                        Q[i + 1] += ch
                    else:
                        lat[e[0]] = max(lat[e[0]], T - e[0] * tau)
                busy[i] = None
        while arrived < X and arrived * tau == T:
            Q[0].append((arrived, 0, None))
            arrived += 1
        for i in decide(T, Q, busy):
            qmax[i] = max(qmax[i], len(Q[i]))
            n = min(len(Q[i]), v)
            ents, Q[i] = Q[i][:n], Q[i][n:]
            busy[i] = (T + t[i], ents)
            if n:
                log.append((i, T, n))
        if arrived == X and not any(Q) and not any(b and b[1] for b in busy):
            _enum_step_semantics.qmax = qmax
            return tuple(lat), log
        T += 1


def _toy_fns():
    gain0 = {0: 1, 1: 0, 2: 2, 3: 1, 4: 1, 5: 0}
    f0 = lambda e: [(e[0], j, None) for j in range(gain0[e[0]])]
    f1 = lambda e: [e]
    return [f0, f1]


def _enumerate_all(N, t, v, tau, X, fns, horizon):
    """Every schedule: at each T each idle node with a non-empty queue fires or waits."""
    out = {}

    def rec(T, Q, busy, lat, arrived, log, act):
        Q = [list(q) for q in Q]
        busy = list(busy)
        lat = list(lat)
        for i in range(N):
            if busy[i] and busy[i][0] == T:
                for e in busy[i][1]:
                    ch = fns[i](e)
                    if i < N - 1 and ch:
                        Q[i + 1] += ch
                    else:
                        lat[e[0]] = max(lat[e[0]], T - e[0] * tau)
                busy[i] = None
        while arrived < X and arrived * tau == T:
            Q[0].append((arrived, 0, None))
            arrived += 1
        if arrived == X and not any(Q) and not any(busy):
            out[tuple(log)] = (tuple(lat), act)
            return
        if T > horizon:
            return
        cand = [i for i in range(N) if busy[i] is None and Q[i]]
        for k in range(len(cand) + 1):
            for fire in itertools.combinations(cand, k):
                Q2 = [list(q) for q in Q]
                b2 = list(busy)
                lg = list(log)
                a2 = act
                for i in fire:
                    n = min(len(Q2[i]), v)
                    b2[i] = (T + t[i], Q2[i][:n])
                    Q2[i] = Q2[i][n:]
                    lg.append((i, T, n))
                    a2 += t[i]
                rec(T + 1, Q2, b2, lat, arrived, lg, a2)

    rec(0, [[] for _ in range(N)], [None] * N, [-1] * X, 0, [], 0)
    return out


@pytest.mark.parametrize("X,tau", [(3, 1), (4, 2)])
def test_p6_schedule_enumeration(X, tau):
    N, t, v = 2, (2, 3), 2
    fns = _toy_fns()
    D = 12
    allsched = _enumerate_all(N, t, v, tau, X, fns, horizon=X * tau + 14)
    assert len(allsched) > 100
    checked = 0
    for policy in (C.FIXED_WAIT, C.THRESHOLD_SLACK):
        params = ([(0, 0), (1, 0), (0, 2), (2, 1), (3, 3)] if policy == C.FIXED_WAIT
                  else [(1, 1), (2, 1), (2, 2), (1, 2)])
        for prm in params:
            cfg = C.Config(name="p6", stages=[C.Stage(C.KEEP_EVERY, 1), C.Stage(C.KEEP_EVERY, 1)],
                           service_time=t, vector_width=v, deadline=D, interarrival=tau, b=(1, 1),
                           wait_time=prm if policy == C.FIXED_WAIT else None,
                           wait_threshold=prm if policy == C.THRESHOLD_SLACK else None,
                           policy=policy, n_roots=X)
            r = des.simulate_stream(cfg, fns, 0, X)
            log = tuple((i, s, n) for (i, s, n, _, _) in r.firings)
            assert log in allsched, (policy, prm, log)
            lat, act = allsched[log]
            assert lat == tuple(r.lat)
            assert act == sum(t[i] for (i, s, n) in log)
            # replay through the independent stepper
            starts = {}
            for (i, s, n) in log:
                starts.setdefault(s, set()).add(i)
            lat2, log2 = _enum_step_semantics(N, t, v, tau, X, fns,
                                              lambda T, Q, b: sorted(starts.get(T, ())))
            assert lat2 == tuple(r.lat) and tuple(log2) == log
            # the queue peaks at firing decisions (L133's b_i v) of the same schedule
            assert _enum_step_semantics.qmax == r.max_queue, (policy, prm)
            # clairvoyant optimum among deadline-meeting schedules is no worse
            ok = [a for (lt, a) in allsched.values() if max(lt) <= D]
            if max(r.lat) <= D:
                assert min(ok) <= act
            checked += 1
    assert checked == 9


def test_monolithic_hand_example():
    """MONOLITHIC (L157, L184): M=2, v=2, t=(2,3), tau=1, 4 roots, gains 1,0,2,1.
    Block 0 = roots {0,1} ready at T=1: node0 fires [1,3) -> children of 0 (1) and 1 (0);
      root 1 terminal at 3; node1 fires [3,6) on {0} -> lat0 = 6.
    Block 1 = roots {2,3} ready at T=3, processor free at 6: node0 [6,8) -> 2 children of
      root 2 + 1 of root 3 = 3 entries; node1 fires [8,11) on 2 entries, [11,14) on 1.
      lat2 = 11 - 2 = 9, lat3 = 14 - 3 = 11."""
    fns = _toy_fns()
    cfg = C.Config(name="mono", stages=[C.Stage(C.KEEP_EVERY, 1), C.Stage(C.KEEP_EVERY, 1)],
                   service_time=(2, 3), vector_width=2, deadline=100, interarrival=1, b=(1, 1),
                   policy=C.MONOLITHIC, block_size=2, n_roots=4)
    r = des.simulate_stream(cfg, fns, 0, 4)
    assert r.lat == [6, 2, 9, 11]
    assert [(i, s, n) for (i, s, n, _, _) in r.firings] == [(0, 1, 2), (1, 3, 1), (0, 6, 2), (1, 8, 2), (1, 11, 1)]
    assert r.T_end == 14


# ------------------------------------------------------------- arrival-time inputs (N2)

def test_explicit_fixed_rate_arrivals_match_default():
    """arrivals[r] = r * tau0 passed as data reproduces the built-in fixed-rate run exactly."""
    for policy in (C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC):
        cfg = gm_cfg(3, (5, 9, 4), (7, 3, 11), 4, 2, 300, seed=4, policy=policy, theta=(3, 2, 4), D=120)
        cfg = cfg.replace(block_size=16)
        a = des.run(cfg)
        b = des.run(cfg, arrivals=[r * 2 for r in range(300)])
        assert (a.lat, a.trace, a.streams[0].firings) == (b.lat, b.trace, b.streams[0].firings)


def _enum_with_arrivals(N, t, v, arr, fns, horizon):
    """Every fire/wait schedule for arbitrary (sorted) arrival times; time-stepped, written
    separately from oracle.des."""
    X = len(arr)
    out = {}

    def rec(T, Q, busy, lat, arrived, log):
        Q = [list(q) for q in Q]
        busy = list(busy)
        lat = list(lat)
        for i in range(N):
            if busy[i] and busy[i][0] == T:
                for e in busy[i][1]:
                    ch = fns[i](e)
                    if i < N - 1 and ch:
                        Q[i + 1] += ch
                    else:
                        lat[e[0]] = max(lat[e[0]], T - arr[e[0]])
                busy[i] = None
        while arrived < X and arr[arrived] == T:
            Q[0].append((arrived, 0, None))
            arrived += 1
        if arrived == X and not any(Q) and not any(busy):
            out[tuple(log)] = tuple(lat)
            return
        if T > horizon:
            return
        cand = [i for i in range(N) if busy[i] is None and Q[i]]
        for k in range(len(cand) + 1):
            for fire in itertools.combinations(cand, k):
                Q2 = [list(q) for q in Q]
                b2 = list(busy)
                lg = list(log)
                for i in fire:
                    n = min(len(Q2[i]), v)
                    b2[i] = (T + t[i], Q2[i][:n])
                    Q2[i] = Q2[i][n:]
                    lg.append((i, T, n))
                rec(T + 1, Q2, b2, lat, arrived, lg)

    rec(0, [[] for _ in range(N)], [None] * N, [-1] * X, 0, [])
    return out


@pytest.mark.parametrize("arr", [(0, 0, 3, 4), (0, 2, 2, 7), (0, 1, 5, 5)])
def test_p6_enumeration_with_arrival_times(arr):
    """P6 with irregular (Poisson-like, simultaneous) arrivals: the DES schedule of each
    policy is one of the enumerated schedules, with identical latencies."""
    N, t, v = 2, (2, 3), 2
    fns = _toy_fns()
    allsched = _enum_with_arrivals(N, t, v, list(arr), fns, horizon=arr[-1] + 16)
    for policy, prm in ((C.FIXED_WAIT, (0, 0)), (C.FIXED_WAIT, (1, 2)), (C.THRESHOLD_SLACK, (2, 1)),
                        (C.THRESHOLD_SLACK, (1, 2))):
        cfg = C.Config(name="p6a", stages=[C.Stage(C.KEEP_EVERY, 1), C.Stage(C.KEEP_EVERY, 1)],
                       service_time=t, vector_width=v, deadline=12, interarrival=2, b=(1, 1),
                       wait_time=prm if policy == C.FIXED_WAIT else None,
                       wait_threshold=prm if policy == C.THRESHOLD_SLACK else None, policy=policy, n_roots=4)
        r = des.simulate_stream(cfg, fns, 0, 4, arrivals=list(arr))
        log = tuple((i, s, n) for (i, s, n, _, _) in r.firings)
        assert log in allsched, (policy, prm, log)
        assert allsched[log] == tuple(r.lat)


# ------------------------------------------------------------- end of stream (R-DRAIN)

@pytest.mark.parametrize("tau,P,t0,v,X", [(4, 128, 64, 32, 97), (3, 10, 7, 4, 23), (5, 5, 5, 1, 9), (2, 9, 1, 8, 40),
                                          (3, 10, 7, 4, 1)])
def test_drain_fixed_wait_single_node_closed_form(tau, P, t0, v, X):
    """R-DRAIN on one FIXED_WAIT node (P <= v tau0): roots whose slot ceil(r tau/P) P precedes
    A_last = (X-1) tau keep P2's latency; the rest leave in one drain firing at
    s = max(A_last, end of the last slot before A_last)."""
    assert P <= v * tau
    cfg = C.Config(name="dr", stages=[C.Stage(C.KEEP_EVERY, 1.0, 1)], service_time=(t0,),
                   vector_width=v, deadline=10**9, interarrival=tau, b=(1,), wait_time=(P - t0,),
                   n_roots=X, eager_drain=True)
    r = des.run(cfg)
    A = (X - 1) * tau
    M = -(-A // P)                                 # slots m P < A_last
    s = max(A, (M - 1) * P + t0) if M else A
    for rr in range(X):
        slot = -(-rr * tau // P)
        expect = slot * P - rr * tau + t0 if slot < M else s + t0 - rr * tau
        assert r.lat[rr] == expect, (rr, r.lat[rr], expect)
    assert r.streams[0].T_end == max(r.lat[rr] + rr * tau for rr in range(X))


@pytest.mark.parametrize("tau,t0,v,X", [(4, 64, 32, 100), (3, 5, 4, 23), (1, 8, 8, 64), (2, 3, 4, 6)])
def test_drain_threshold_single_node_closed_form(tau, t0, v, X):
    """R-DRAIN on one THRESHOLD_SLACK node (theta = v, no slack force): full groups fire at
    their v-th arrival; the last partial group at max(A_last, end of the last full group)."""
    D = 10**6
    assert t0 <= v * tau
    cfg = C.Config(name="drt", stages=[C.Stage(C.KEEP_EVERY, 1.0, 1)], service_time=(t0,),
                   vector_width=v, deadline=D, interarrival=tau, b=(1,), wait_threshold=(v,),
                   policy=C.THRESHOLD_SLACK, n_roots=X, eager_drain=True)
    r = des.run(cfg)
    full = (X // v) * v
    for rr in range(full):
        assert r.lat[rr] == (v - 1 - rr % v) * tau + t0
    s = max((X - 1) * tau, (full - 1) * tau + t0 if full else 0)
    for rr in range(full, X):
        assert r.lat[rr] == s + t0 - rr * tau


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_drain_changes_nothing_before_last_arrival(policy, seed):
    """R-DRAIN acts only at T >= A_last: every firing that starts earlier is identical, and
    the invariants of P4 hold throughout."""
    rnd = random.Random(seed)
    N = rnd.randint(2, 4)
    t = [rnd.randint(3, 30) for _ in range(N)]
    cfg = gm_cfg(N, t, [rnd.randint(0, 50) for _ in range(N)], rnd.choice([4, 8]), rnd.randint(1, 6),
                 rnd.randint(50, 300), seed=seed, policy=policy,
                 theta=[rnd.randint(1, 4) for _ in range(N)], D=rnd.randint(100, 400))
    a = des.run(cfg)
    b = des.run(cfg.replace(eager_drain=True), check_invariants=True)
    A = (cfg.n_roots - 1) * cfg.interarrival
    fa = [f for f in a.streams[0].firings if f[1] < A]
    fb = [f for f in b.streams[0].firings if f[1] < A]
    assert fa == fb
    assert b.matches == a.matches and b.trace == a.trace          # the data path does not depend on it
    assert b.streams[0].T_end <= a.streams[0].T_end


@pytest.mark.parametrize("X,tau", [(3, 1), (4, 2)])
def test_drain_schedule_enumeration(X, tau):
    """P6 for R-DRAIN: the DES schedule is one of the enumerated fire/wait schedules, and the
    independent stepper driven by the rule written out here reproduces it exactly."""
    N, t, v = 2, (2, 3), 2
    fns = _toy_fns()
    D = 12
    A = (X - 1) * tau
    allsched = _enumerate_all(N, t, v, tau, X, fns, horizon=X * tau + 14)
    for policy in (C.FIXED_WAIT, C.THRESHOLD_SLACK):
        params = ([(0, 0), (1, 0), (0, 2), (2, 1), (3, 3)] if policy == C.FIXED_WAIT
                  else [(1, 1), (2, 1), (2, 2), (1, 2)])
        for prm in params:
            cfg = C.Config(name="p6d", stages=[C.Stage(C.KEEP_EVERY, 1), C.Stage(C.KEEP_EVERY, 1)],
                           service_time=t, vector_width=v, deadline=D, interarrival=tau, b=(1, 1),
                           wait_time=prm if policy == C.FIXED_WAIT else None,
                           wait_threshold=prm if policy == C.THRESHOLD_SLACK else None,
                           policy=policy, n_roots=X, eager_drain=True)
            r = des.simulate_stream(cfg, fns, 0, X)
            log = tuple((i, s, n) for (i, s, n, _, _) in r.firings)
            assert log in allsched, (policy, prm, log)
            assert allsched[log][0] == tuple(r.lat)
            if policy == C.FIXED_WAIT:
                P = [t[i] + prm[i] for i in range(N)]
                rule = lambda T, Q, b: [i for i in range(N)
                                        if (T < A and T % P[i] == 0) or (T >= A and b[i] is None and Q[i])]
            else:
                R = [t[0] + 2 * t[1], t[1]]
                rule = lambda T, Q, b: [i for i in range(N) if b[i] is None and Q[i] and (
                    len(Q[i]) >= prm[i] or T >= Q[i][0][0] * tau + D - R[i] or T >= A)]
            lat2, log2 = _enum_step_semantics(N, t, v, tau, X, fns, rule)
            assert lat2 == tuple(r.lat) and tuple(log2) == log, (policy, prm)
