"""Discrete-event simulation of the paper's execution model (ORACLE — test infrastructure).

Follows PAPER.md §2 (application model L59–L63, implementation model L65–L69,
criteria L71–L77), §4 (enforced waiting, L95–L97) and §5 (monolithic, L157,
L184), step by step, in integer time, as written out in SURVEY.md §8(c) C-D and
DESIGN.md "Readings".  Plain Python: one heap of integer event times, one deque
per edge, per-item stage evaluation through ``oracle.stages``.

At each event time T, in this order (reading R-ORDER):
  1. completions (node 0..N-1): children of every consumed entry, in lane order
     then child order, are appended to Q[i+1] with ready = T (R-VISIBLE, A9);
     an entry with no children, or consumed by node N-1, is terminal and sets
     lat[r] = max(lat[r], T - a(r))  (R-DONE, A12; deadline L73);
  2. arrivals with r*tau0 == T are appended to Q[0]  (L63);
  3. starts, by policy:
       FIXED_WAIT      — node i fires at every m*(t_i+w_i) (phase 0, R-PHASE),
                         taking min(|Q_i|, v) head entries, charged t_i even when
                         empty  (L97);
       THRESHOLD_SLACK — an idle node fires when |Q_i| >= theta_i or when
                         |Q_i| > 0 and T >= a(head) + D - R_i (north_star rule,
                         SURVEY A25), taking min(|Q_i|, v);
     With ``cfg.eager_drain`` (reading R-DRAIN): at every event time
     T >= A_last (the stream's last arrival) both policies give way to a
     work-conserving drain -- an idle node with a non-empty queue fires at T,
     taking min(|Q_i|, v); FIXED_WAIT's time-triggered starts at T >= A_last are
     dropped.  Before A_last nothing changes.
  4. stop once every root has arrived, every queue is empty and no firing
     with inputs is in flight (FIXED_WAIT also keeps generating its
     time-triggered firings until every node's next start is >= H = X*tau0, so
     that the window [0, H) is fully charged, R-WINDOW; with eager_drain there
     are none at T >= A_last).
MONOLITHIC (L157, L184; R-MONO) is simulated by its own loop: blocks of M
consecutive arrivals, ready at their last arrival, served FIFO by one
processor; for each block node i fires ceil(n_i/v) times back to back.
"""
from __future__ import annotations

import dataclasses
import heapq
from collections import deque

from plgen import configs as C
from plgen import gaintab
from . import stages as S


@dataclasses.dataclass
class StreamResult:
    lo: int
    hi: int
    lat: list            # per local root (int)
    trace: list          # flat, (hi-lo) x (N+1)
    matches: list        # DNA: HSP tuples; gain model: []
    firings: list        # (node, start, n, first_root, last_root) for firings with n > 0
    n_firings: list      # per node, all firings incl. empty, started before stop
    n_empty: list
    consumed: list
    produced: list
    active_H: list       # per node: sum |[s, s+t_i) ∩ [0, H)| over all firings
    active_H_nonempty: list
    active_drain: list   # per node: sum |[s, s+t_i) ∩ [0, T_end)| over firings with s < T_end
    H: int
    T_end: int
    max_queue: list = None   # per node: max |Q_i| at its firing decisions ("maximum
                             # size b_i v"), counted before the firing takes its inputs


def gains_G(g):
    """G_0 = 1, G_i = prod_{j<i} g_j  (garbled; reading A1)."""
    G = [1.0]
    for x in g:
        G.append(G[-1] * x)
    return G


def reserve(t, i):
    """R_i = t_i + 2 * sum_{j>i} t_j (THRESHOLD_SLACK slack reserve; the config's
    slack_guard is added on top, DESIGN.md R-THRESH)."""
    return t[i] + 2 * sum(t[i + 1:])


def make_stage_fns(cfg: C.Config, ctx: S.DnaContext | None):
    fns = []
    for i, st in enumerate(cfg.stages):
        k = st.kind
        if k == C.BERNOULLI:
            thr = gaintab.bernoulli_table(st.param)[0]
            fns.append(lambda e, i=i, thr=thr: S.g_bernoulli(cfg.seed, i, e, thr))
        elif k == C.FIXED_GAIN:
            c = int(st.param)
            fns.append(lambda e, c=c: S.g_fixed(e, c))
        elif k == C.POISSON_CAPPED:
            tab = gaintab.poisson_capped_table(st.param, st.max_out)
            fns.append(lambda e, i=i, tab=tab, u=st.max_out: S.g_poisson_capped(cfg.seed, i, e, tab, u))
        elif k == C.KEEP_EVERY:
            fns.append(lambda e, m=int(st.param): S.g_keep_every(e, m))
        elif k == C.SEED_LOOKUP:
            fns.append(lambda e: S.s0_seed_lookup(ctx, e))
        elif k == C.HIT_ENUM:
            fns.append(lambda e, u=st.max_out: S.s1_hit_enum(ctx, e, u))
        elif k == C.UNGAPPED_WINDOW:
            fns.append(lambda e, W=st.iparam[1], T2=st.iparam[2]: S.s2_window(ctx, e, W, T2))
        elif k == C.UNGAPPED_XDROP:
            fns.append(lambda e, X=st.iparam[1], T3=st.iparam[2]: S.s3_xdrop(ctx, e, X, T3))
        else:
            raise ValueError(f"unknown stage kind {k}")
    return fns


def _overlap(s, e, lo, hi):
    return max(0, min(e, hi) - max(s, lo))


def simulate_stream(cfg: C.Config, fns, lo: int, hi: int, wait_time=None, theta=None,
                    block_size=None, check_invariants=False, node_order=None, arrivals=None) -> StreamResult:
    """Simulate one independent stream whose roots are the global ids [lo, hi).

    Root r (global) arrives at a(r) = (r - lo) * tau0, or at arrivals[r - lo]
    when an arrival-time array is given (non-decreasing; Poisson arrivals, L263).
    ``node_order`` permutes the order in which nodes are visited inside phases 1 and 3 (pin P5).
    """
    if cfg.policy == C.MONOLITHIC:
        return _simulate_monolithic(cfg, fns, lo, hi, block_size, arrivals)
    N = cfg.n_stages
    t = list(cfg.service_time)
    v = cfg.vector_width
    tau = cfg.interarrival
    D = cfg.deadline
    X = hi - lo
    H = X * tau
    arr = [r * tau for r in range(X)] if arrivals is None else [int(x) for x in arrivals]
    order = list(range(N)) if node_order is None else list(node_order)
    match_sink = cfg.stages[-1].kind == C.UNGAPPED_XDROP
    fixed = cfg.policy == C.FIXED_WAIT
    eager = bool(getattr(cfg, "eager_drain", False))
    A_last = arr[X - 1] if X else 0              # R-DRAIN: the drain starts at the last arrival
    if fixed:
        w = list(wait_time if wait_time is not None else cfg.wait_time)
        P = [t[i] + w[i] for i in range(N)]
        next_start = [0] * N                     # phase 0 for every node (R-PHASE)
    else:
        th = list(theta if theta is not None else cfg.wait_threshold)
        R = [reserve(t, i) + getattr(cfg, "slack_guard", 0) for i in range(N)]
        last_force = [None] * N

    Q = [deque() for _ in range(N)]              # entries (root, lin, q)
    inflight = [None] * N                        # (start, end, [entries])
    lat = [-1] * X
    trace = [0] * (X * (N + 1))
    matches = []
    firings = []
    starts = [[] for _ in range(N)]              # every firing start (incl. empty)
    n_firings = [0] * N
    n_empty = [0] * N
    consumed = [0] * N
    produced = [0] * N
    active_H = [0] * N
    active_H_ne = [0] * N
    max_queue = [0] * N
    T_end = 0
    next_root = 0
    heap = [0] + ([arr[0]] if X else [])
    last_T = None
    entered = [0] * N                            # for invariant checks (P4)

    def push(x):
        heapq.heappush(heap, x)

    while heap:
        T = heapq.heappop(heap)
        if T == last_T:
            continue
        last_T = T
        # ---- 1. completions
        for i in order:
            f = inflight[i]
            if f is None or f[1] != T:
                continue
            inflight[i] = None
            for e in f[2]:
                ch = fns[i](e)
                r = e[0] - lo
                produced[i] += len(ch)
                if i == N - 1:
                    trace[r * (N + 1) + N] += len(ch)
                    if match_sink:
                        matches.extend(ch)
                    lat[r] = max(lat[r], T - arr[r])
                elif ch:
                    Q[i + 1].extend(ch)
                    entered[i + 1] += len(ch)
                else:
                    lat[r] = max(lat[r], T - arr[r])
            if f[2]:
                T_end = max(T_end, T)
        # ---- 2. arrivals
        if next_root < X and arr[next_root] == T:
            while next_root < X and arr[next_root] == T:
                Q[0].append((lo + next_root, 0, None))
                entered[0] += 1
                next_root += 1
            if next_root < X:
                push(arr[next_root])
        # ---- 3. starts
        for i in order:
            fire = False
            if eager and T >= A_last:                # R-DRAIN: work-conserving after the last arrival
                fire = inflight[i] is None and bool(Q[i])
            elif fixed:
                fire = next_start[i] == T
            elif inflight[i] is None and Q[i]:
                a_head = arr[Q[i][0][0] - lo]
                fire = len(Q[i]) >= th[i] or T >= a_head + D - R[i]
            if fire:
                max_queue[i] = max(max_queue[i], len(Q[i]))
                n = min(len(Q[i]), v)
                ents = [Q[i].popleft() for _ in range(n)]
                for e in ents:
                    trace[(e[0] - lo) * (N + 1) + i] += 1
                consumed[i] += n
                inflight[i] = (T, T + t[i], ents)
                push(T + t[i])
                n_firings[i] += 1
                starts[i].append(T)
                ov = _overlap(T, T + t[i], 0, H)
                active_H[i] += ov
                if n:
                    active_H_ne[i] += ov
                    firings.append((i, T, n, ents[0][0], ents[-1][0]))
                else:
                    n_empty[i] += 1
                if fixed and not (eager and T + P[i] >= A_last):
                    next_start[i] = T + P[i]
                    push(next_start[i])
                elif fixed:
                    next_start[i] = 1 << 62          # no time-triggered starts at or after A_last
            if not fixed and Q[i]:
                fdl = arr[Q[i][0][0] - lo] + D - R[i]
                if fdl > T and last_force[i] != fdl:
                    last_force[i] = fdl
                    push(fdl)
        if check_invariants:
            _check_conservation(N, entered, consumed, Q, produced, next_root, X, trace, lat)
        # ---- 4. stop
        drained = (next_root == X and all(not q for q in Q)
                   and all(f is None or not f[2] for f in inflight))
        if drained and (not fixed or min(next_start) >= H):
            break

    active_drain = [sum(_overlap(s, s + t[i], 0, T_end) for s in starts[i] if s < T_end)
                    for i in range(N)]
    return StreamResult(lo, hi, lat, trace, matches, firings, n_firings, n_empty, consumed,
                        produced, active_H, active_H_ne, active_drain, H, T_end, max_queue)


def _check_conservation(N, entered, consumed, Q, produced, next_root, X, trace, lat):
    """Pin P4 (north_star conservation), after every event time:
    entered_i = consumed_i + queued_i; produced_i = entered_{i+1};
    sum_r cnt[r][i] = consumed_i; arrived roots = completed + pending."""
    assert entered[0] == next_root <= X
    for i in range(N):
        assert entered[i] == consumed[i] + len(Q[i]), (i, entered[i], consumed[i], len(Q[i]))
        if i + 1 < N:
            assert produced[i] == entered[i + 1], (i, produced[i], entered[i + 1])
        assert sum(trace[r * (N + 1) + i] for r in range(X)) == consumed[i]
    done = sum(1 for x in lat if x >= 0)
    assert done <= next_root


def _simulate_monolithic(cfg, fns, lo, hi, M, arrivals=None):
    """MONOLITHIC (§5; reading R-MONO)."""
    N = cfg.n_stages
    t = list(cfg.service_time)
    v = cfg.vector_width
    tau = cfg.interarrival
    X = hi - lo
    H = X * tau
    M = int(M if M is not None else cfg.block_size)
    arr = [r * tau for r in range(X)] if arrivals is None else [int(x) for x in arrivals]
    lat = [-1] * X
    trace = [0] * (X * (N + 1))
    matches = []
    firings = []
    n_firings = [0] * N
    consumed = [0] * N
    produced = [0] * N
    active_H = [0] * N
    starts = [[] for _ in range(N)]
    proc_free = 0
    T_end = 0
    for b0 in range(0, X, M):
        b1 = min(b0 + M, X)
        ready = arr[b1 - 1]                      # last root of the block has arrived
        T = max(ready, proc_free)
        cur = [(lo + r, 0, None) for r in range(b0, b1)]
        for i in range(N):
            nxt = []
            for f0 in range(0, len(cur), v):
                ents = cur[f0:f0 + v]
                s, e_ = T, T + t[i]
                T = e_
                n_firings[i] += 1
                consumed[i] += len(ents)
                starts[i].append(s)
                active_H[i] += _overlap(s, e_, 0, H)
                firings.append((i, s, len(ents), ents[0][0], ents[-1][0]))
                for e in ents:
                    r = e[0] - lo
                    trace[r * (N + 1) + i] += 1
                    ch = fns[i](e)
                    produced[i] += len(ch)
                    if i == N - 1:
                        trace[r * (N + 1) + N] += len(ch)
                        if cfg.stages[-1].kind == C.UNGAPPED_XDROP:
                            matches.extend(ch)
                        lat[r] = max(lat[r], e_ - arr[r])
                    elif ch:
                        nxt.extend(ch)
                    else:
                        lat[r] = max(lat[r], e_ - arr[r])
                T_end = max(T_end, e_)
            cur = nxt
        proc_free = T
    active_drain = [sum(_overlap(s, s + t[i], 0, T_end) for s in starts[i] if s < T_end)
                    for i in range(N)]
    return StreamResult(lo, hi, lat, trace, matches, firings, n_firings, [0] * N, consumed,
                        produced, active_H, list(active_H), active_drain, H, T_end, [0] * N)


# ------------------------------------------------------------------ drivers

@dataclasses.dataclass
class Result:
    streams: list
    lat: list
    trace: list
    matches: list
    N: int

    def max_queue(self):
        """Per node: the longest input queue over all streams at a firing decision."""
        return [max((s.max_queue[i] for s in self.streams), default=0) for i in range(self.N)]

    def misses(self, D):
        return sum(1 for x in self.lat if x > D)

    def max_lat(self):
        return max(self.lat) if self.lat else 0

    def active_fraction(self, policy, nonempty=False):
        """Active / (active + waiting) over [0, H) (reading R-WINDOW).
        Enforced policies: (1/(N H)) sum_i active_i; monolithic: (1/H) sum_i busy_i."""
        acc = sum(sum(s.active_H_nonempty if nonempty else s.active_H) for s in self.streams)
        H = sum(s.H for s in self.streams)
        return acc / H if policy == C.MONOLITHIC else acc / (self.N * H)

    def active_fraction_drain(self, policy):
        """The same ratio over [0, T_end] (the drain included; SURVEY §8(c) C-D "Outputs"):
        every firing that starts before T_end, clipped to it, over N T_end (enforced) or
        T_end (monolithic), summed over streams.  Pinned by test_oracle_des.py::
        test_p1_drain_window_closed_form (FIXED_WAIT charges every slot m P_i < T_end)."""
        acc = sum(sum(s.active_drain) for s in self.streams)
        Te = sum(s.T_end for s in self.streams)
        return acc / Te if policy == C.MONOLITHIC else acc / (self.N * Te)


def stream_ranges(cfg: C.Config, n_roots_total: int):
    S = cfg.n_streams
    return [((s * n_roots_total) // S, ((s + 1) * n_roots_total) // S) for s in range(S)]


def run(cfg: C.Config, workload=None, streams=None, arrivals=None, **kw) -> Result:
    """Simulate every stream of ``cfg`` (or the subset ``streams``) and merge.

    DNA configs need ``workload`` (plgen.dna.DnaWorkload); roots are DB
    positions [0, Ldb-k].  Gain-model configs have n_roots * n_streams roots.
    """
    ctx = None
    if cfg.stages[0].kind in C.DNA_KINDS:
        k = cfg.stages[0].iparam[0]
        ctx = S.DnaContext(workload.db, workload.db_len, workload.query, workload.q_len, k)
        total = ctx.n_roots
    else:
        total = cfg.n_roots * cfg.n_streams
    fns = make_stage_fns(cfg, ctx)
    rng = stream_ranges(cfg, total)
    idx = range(len(rng)) if streams is None else streams
    res = [simulate_stream(cfg, fns, rng[s][0], rng[s][1],
                           arrivals=None if arrivals is None else arrivals[rng[s][0]:rng[s][1]], **kw) for s in idx]
    lat, trace, matches = [], [], []
    for r in res:
        lat += r.lat
        trace += r.trace
        matches += r.matches
    matches.sort()
    return Result(res, lat, trace, matches, cfg.n_stages)
