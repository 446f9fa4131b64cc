"""CLI / timing harness of the oracle (ORACLE — test infrastructure; used by bench.py's
``cpu_baseline`` and ``--impl reference`` legs only).

    python -m oracle.run --config c4 --procs 8 --streams 16 --roots 20000

runs ``oracle.des.simulate_stream`` -- the plain discrete-event simulation, as it stands --
over a bounded sample of the configuration's streams (the first ``--roots`` roots of each of
``--streams`` streams) in a fork process pool, and prints one JSON line with the sample, the
wall time and the oracle's items/s.  Nothing here computes the method beyond calling the DES.
"""
from __future__ import annotations

import argparse
import json
import math
import multiprocessing as mp
import os
import time

from plgen import configs as C
from plgen import dna as G
from . import des
from . import solver as SV
from . import stages as S

_CTX = {}


def _one(args):
    cfg, lo, hi = args
    fns = des.make_stage_fns(cfg, _CTX.get("ctx"))   # the context is built once, before the fork
    r = des.simulate_stream(cfg, fns, lo, hi)
    return hi - lo, max(r.lat) if r.lat else 0


def sample_ranges(cfg, wl, n_streams, max_roots):
    """The first ``max_roots`` roots of the first ``n_streams`` streams of the configuration."""
    if wl is not None:
        total = wl.db_len - cfg.stages[0].iparam[0] + 1
    else:
        total = cfg.n_roots * cfg.n_streams
    rng = des.stream_ranges(cfg, total)[:n_streams]
    return [(lo, min(hi, lo + max_roots) if max_roots else hi) for lo, hi in rng]


def time_oracle(cfg, wl, n_streams, max_roots=0, procs=None):
    """Wall-clock the DES over the sample on ``procs`` host processes.
    Returns dict(value items/s, cores, seconds, roots, sample)."""
    if _CTX.get("wl") is not wl:
        _CTX["wl"] = wl
        _CTX["ctx"] = (S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, cfg.stages[0].iparam[0])
                       if wl is not None else None)
    ranges = sample_ranges(cfg, wl, n_streams, max_roots)
    cores = procs or len(os.sched_getaffinity(0))
    t0 = time.perf_counter()
    if cores == 1:
        res = [_one((cfg, lo, hi)) for lo, hi in ranges]
    else:
        with mp.get_context("fork").Pool(min(cores, len(ranges))) as pool:
            res = pool.map(_one, [(cfg, lo, hi) for lo, hi in ranges], chunksize=1)
    dt = time.perf_counter() - t0
    roots = sum(r[0] for r in res)
    return {"value": roots / dt if dt > 0 else 0.0, "cores": min(cores, len(ranges)), "seconds": dt,
            "roots": roots, "sample": f"{len(ranges)} streams x first {max_roots or 'all'} roots"}


def oracle_schedule(cfg, gains=None):
    """FIXED_WAIT waits from the oracle's own Fig. 1 solver: the continuous optimum (SLSQP)
    floored to integers and checked feasible, as tests/test_oracle_paper_stats.py does.
    ``gains`` default to Table 1."""
    g = tuple(gains) if gains is not None else (tuple(cfg.gain) if cfg.gain is not None else C.TABLE1_G)
    N = cfg.n_stages
    Pc, _ = SV.fig1_continuous(cfg.service_time, g, cfg.b, cfg.vector_width, cfg.interarrival, cfg.deadline)
    if Pc is None:
        raise RuntimeError("Fig. 1 infeasible")
    # floored, then repaired down the chain so that g_{i-1} P_i <= P_{i-1} holds in integers
    P = [max(cfg.service_time[0], min(math.floor(Pc[0]), cfg.vector_width * cfg.interarrival))]
    for i in range(1, N):
        P.append(max(cfg.service_time[i], min(math.floor(Pc[i]), math.floor(P[i - 1] / g[i - 1]))))
    if not SV.fig1_feasible(cfg.service_time, g, cfg.b, cfg.vector_width, cfg.interarrival, cfg.deadline, P):
        raise RuntimeError("floored Fig. 1 point infeasible")
    w = tuple(P[i] - cfg.service_time[i] for i in range(N))
    th = tuple(SV.thresholds(g, P, cfg.interarrival, cfg.vector_width))
    return cfg.replace(wait_time=w, wait_threshold=th, gain=g)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2", choices=["c1", "c2", "c4"])
    ap.add_argument("--procs", type=int, default=None)
    ap.add_argument("--streams", type=int, default=16)
    ap.add_argument("--roots", type=int, default=0, help="roots per stream (0 = whole stream)")
    ap.add_argument("--policy", type=int, default=C.FIXED_WAIT)
    ap.add_argument("--n-streams", type=int, default=148, help="streams the workload is split into")
    a = ap.parse_args()
    base = getattr(C, a.config)()
    if base.dna:
        base = base.replace(n_streams=a.n_streams)
    wl = G.make_dna(base.seed, **base.dna) if base.dna else None
    cfg = oracle_schedule(base.replace(policy=a.policy))
    print(json.dumps(dict(time_oracle(cfg, wl, a.streams, a.roots, a.procs), config=a.config)))


if __name__ == "__main__":
    main()
