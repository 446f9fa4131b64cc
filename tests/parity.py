"""Shared helpers for the GPU parity tests: run the CUDA path (through the C-ABI)
and the oracle on the same seeded inputs and compare element by element."""
from __future__ import annotations

import numpy as np

from plgen import configs as C
from plgen import dna as G


def workload_for(cfg):
    if cfg.dna is None:
        return None
    return G.make_dna(cfg.seed, **cfg.dna)


def run_gpu(cfg, wl, flags=7, arrivals=None, **over):
    from paper_conf_icppw_planob21_b200 import Pipeline
    pl = Pipeline(cfg, wl, flags=flags, arrivals=arrivals, **over)
    if wl is not None:
        pl.push(wl.db, wl.db_len)
    else:
        pl.push(None, cfg.n_roots)
    pl.drain()
    out = dict(stats=pl.stats(), matches=pl.results() if wl is not None else [])
    if flags & 1:
        out["lat"], out["lat_ns"] = pl.latency()
    if flags & 2:
        out["trace"] = pl.trace()
    if flags & 4:
        out["firings"] = pl.firings()
    out["params"] = pl.params()
    pl.close()
    return out


def run_oracle(cfg, wl, streams=None, arrivals=None):
    from oracle import des
    return des.run(cfg, wl, streams=streams, arrivals=arrivals)


def oracle_firings(res, stream_ids=None):
    out = []
    for k, s in enumerate(res.streams):
        sid = stream_ids[k] if stream_ids is not None else k
        for (i, st, n, a, b) in s.firings:
            out.append((sid, i, st, n, a, b))
    return sorted(out)


def compare(cfg, g, o, check_firings=True):
    """Assert bit-exact agreement of everything the logical schedule determines."""
    N = cfg.n_stages
    st = g["stats"]
    assert st["errors"] == 0, st["errors"]
    assert g["matches"] == [tuple(m) for m in o.matches]
    if "lat" in g:
        assert np.array_equal(g["lat"], np.asarray(o.lat, dtype=np.int64))
    if "trace" in g:
        assert np.array_equal(g["trace"], np.asarray(o.trace, dtype=np.uint32))
    if check_firings and "firings" in g:
        assert sorted(g["firings"]) == oracle_firings(o)
    for i in range(N):
        assert st["consumed"][i] == sum(s.consumed[i] for s in o.streams), i
        assert st["produced"][i] == sum(s.produced[i] for s in o.streams), i
        ne = sum(1 for s in o.streams for f in s.firings if f[0] == i)
        assert st["firings"][i] == ne, i
        assert st["active_window"][i] == sum(s.active_H[i] for s in o.streams), i
    assert st["t_end"] == sum(s.T_end for s in o.streams)
    assert st["max_latency"] == max(o.lat)
    if cfg.clock == C.CLOCK_LOGICAL:
        assert st["misses"] == o.misses(cfg.deadline)
    elif "lat" in g:       # physical: pl_stats.misses counts measured latencies; the schedule's are exact
        assert int((g["lat"] > cfg.deadline).sum()) == o.misses(cfg.deadline)
    assert abs(st["active_fraction"] - o.active_fraction(cfg.policy)) < 1e-12
    # the vacation reading of L97 (non-empty firings only) and the drain-inclusive ratio
    assert abs(st["active_fraction_nonempty"] - o.active_fraction(cfg.policy, nonempty=True)) < 1e-12
    assert abs(st["active_fraction_drain"] - o.active_fraction_drain(cfg.policy)) < 1e-12
    # queue peaks at firing decisions (L133's b_i v): exact on the logical clock, where a node
    # commits before its upstream watermark passes T only when the producer is stalled
    if cfg.policy != C.MONOLITHIC and cfg.clock == C.CLOCK_LOGICAL and sum(st["stalls"]) == 0:
        assert st["max_queue"] == o.max_queue(), (st["max_queue"], o.max_queue())


_WL = None


def _oracle_one(args):
    cfg, lo, hi, kw = args
    from oracle import des
    from oracle import stages as S
    ctx = None
    if _WL is not None:
        ctx = S.DnaContext(_WL.db, _WL.db_len, _WL.query, _WL.q_len, cfg.stages[0].iparam[0])
    fns = des.make_stage_fns(cfg, ctx)
    return des.simulate_stream(cfg, fns, lo, hi, **kw)


def run_oracle_parallel(cfg, wl, streams=None, **kw):
    """oracle.des.run over a fork process pool (same result as run_oracle)."""
    global _WL
    import multiprocessing as mp
    import os
    from oracle import des
    _WL = wl
    if wl is not None:
        total = wl.db_len - cfg.stages[0].iparam[0] + 1
    else:
        total = cfg.n_roots * cfg.n_streams
    rng = des.stream_ranges(cfg, total)
    idx = list(range(len(rng))) if streams is None else list(streams)
    with mp.get_context("fork").Pool(min(len(idx), len(os.sched_getaffinity(0)))) as pool:
        res = pool.map(_oracle_one, [(cfg, rng[s][0], rng[s][1], kw) for s in idx], chunksize=1)
    lat, trace, matches = [], [], []
    for r in res:
        lat += r.lat
        trace += r.trace
        matches += r.matches
    matches.sort()
    return des.Result(res, lat, trace, matches, cfg.n_stages)
