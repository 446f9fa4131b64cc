"""GPU parity of live ingest (a1; §2.1 "a stream of items, of unbounded length").

One persistent run executes while the host delivers the DB: pl_pipeline_live_start launches it,
pl_pipeline_push_stream / push_all append each stream's words to its device ring (the copy stream
rings the stream's doorbell behind the words), node 0 takes a root only once every word its
descendants can read has arrived, and ring slots are reused once the device publishes that no
node reads below them.  The logical schedule is the oracle's whatever the delivery timing, so
every parity output must be bit-exact -- here with rings far shorter than the streams (each slot
rewritten several times), deliveries slower than the executor, and all three policies.
"""
import time

import numpy as np
import pytest

from plgen import configs as C
from parity import compare, run_oracle, workload_for

pytestmark = pytest.mark.gpu


def _dna(policy, db_len=1 << 16, streams=2, **kw):
    cfg = C.c2(n_streams=streams, dna=dict(db_len=db_len, q_len=1024, n_planted=16), **kw)
    if policy == C.FIXED_WAIT:
        return cfg.replace(wait_time=(993, 2422, 965, 1628))
    if policy == C.THRESHOLD_SLACK:
        return cfg.replace(policy=policy, wait_threshold=(128, 127, 99, 10))
    return cfg.replace(policy=policy, block_size=2688)


def deliver(pl, wl, S, slice_words, pause=0.0, per_stream=False):
    """Push every stream's words [lo, hi) in slices of `slice_words`, pausing between slices."""
    rng = [pl.stream_words(s) for s in range(S)]
    pos = [lo for lo, _ in rng]
    pushes = 0
    while any(pos[s] < rng[s][1] for s in range(S)):
        sl = []
        for s in range(S):
            e = min(pos[s] + slice_words, rng[s][1])
            sl.append(wl.db[pos[s]:e])
            pos[s] = e
        if per_stream:
            for s in range(S):
                if len(sl[s]):
                    pl.push_stream(s, sl[s])
        else:
            pl.push_all(sl)
        pushes += 1
        if pause:
            time.sleep(pause)
    return pushes


def run_live(cfg, wl, flags=7, ring_words=0, slice_words=97, pause=0.0, per_stream=False, **over):
    from paper_conf_icppw_planob21_b200 import Pipeline
    pl = Pipeline(cfg, wl, flags=flags, **over)
    pl.live_start(ring_words)
    deliver(pl, wl, cfg.n_streams, slice_words, pause, per_stream)
    pl.drain()
    out = dict(stats=pl.stats(), matches=pl.results())
    if flags & 1:
        out["lat"], out["lat_ns"] = pl.latency()
    if flags & 2:
        out["trace"] = pl.trace()
    if flags & 4:
        out["firings"] = pl.firings()
    pl.close()
    return out


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_live_logical_small_rings(policy):
    """2 streams of 32 K roots (~2.2 K words each) through 512-word rings behind a 256-word smem
    window: every ring slot is rewritten ~4 times while the run executes; bit-exact."""
    cfg = _dna(policy)
    wl = workload_for(cfg)
    g = run_live(cfg, wl, ring_words=512, window_words=256, window_chunk_words=64, slice_words=61)
    st = g["stats"]
    assert st["window_refills"] > 0
    compare(cfg, g, run_oracle(cfg, wl))


@pytest.mark.parametrize("per_stream", [False, True])
def test_live_logical_slow_delivery(per_stream):
    """Deliveries slower than the executor (a pause after every slice): node 0 waits for words
    (pl_stats.ingest_waits > 0) and the results do not move."""
    cfg = _dna(C.THRESHOLD_SLACK, streams=5)
    wl = workload_for(cfg)
    g = run_live(cfg, wl, slice_words=128, pause=0.002, per_stream=per_stream)
    assert g["stats"]["ingest_waits"] > 0
    compare(cfg, g, run_oracle(cfg, wl))


def test_live_physical_paced_delivery():
    """The %globaltimer clock with the host delivering each slice about when its roots arrive:
    the logical schedule (matches, traces, model latencies, firing log) is bit-exact; measured
    latencies include any delivery lateness."""
    cfg = _dna(C.THRESHOLD_SLACK, streams=4).replace(clock=C.CLOCK_GLOBALTIMER, ns_per_unit=1.0,
                                                     service_time=(20_000,) * 4, interarrival=400,
                                                     deadline=10_000_000)
    wl = workload_for(cfg)
    # one slice = 64 words = 1024 roots = 410 us of arrivals per stream
    g = run_live(cfg, wl, slice_words=64, pause=0.0004)
    st = g["stats"]
    assert st["errors"] == 0
    compare(cfg, g, run_oracle(cfg, wl))
    assert (g["lat_ns"] > 0).all()
    print("ingest waits", st["ingest_waits"], "max wait ns", st["max_ingest_wait_ns"],
          "lateness", st["max_lateness_ns"])


def test_live_errors_and_backpressure():
    from paper_conf_icppw_planob21_b200 import Pipeline
    from paper_conf_icppw_planob21_b200._pl import PL_EAGAIN, PL_EINVAL, PL_ESTATE, PlError
    cfg = _dna(C.THRESHOLD_SLACK)
    wl = workload_for(cfg)
    pl = Pipeline(cfg, wl, window_words=256, window_chunk_words=64)
    lo, hi = pl.stream_words(0)
    with pytest.raises(PlError) as e:            # no live run yet
        pl.push_stream(0, wl.db[lo:lo + 16])
    assert e.value.status == PL_ESTATE
    pl.live_start(512)
    with pytest.raises(PlError) as e:            # more than the ring holds, non-blocking
        pl.push_stream(0, wl.db[lo:lo + 600], nonblocking=True)
    assert e.value.status == PL_EAGAIN
    with pytest.raises(PlError) as e:            # past the stream's range
        pl.push_stream(1, np.zeros(1 << 20, dtype=np.uint32))
    assert e.value.status == PL_EINVAL
    with pytest.raises(PlError) as e:            # a launch while the live run executes
        pl.launch()
    assert e.value.status == PL_ESTATE
    with pytest.raises(PlError) as e:            # drain before every word was pushed
        pl.drain()
    assert e.value.status == PL_ESTATE
    deliver(pl, wl, cfg.n_streams, 100)
    pl.drain()
    assert pl.stats()["errors"] == 0
    pl.close()


def test_live_c4_sampled_streams():
    """c4 at full size (148 streams x 708 K roots, 100 Mbp, heavy-tailed) delivered live in
    slices through 64 K-word rings, logical clock: matches of sampled streams bit-exact vs the
    oracle's prefix DES and the match count equal to a bound-DB run's."""
    import torch
    from oracle import des
    from oracle import stages as S
    from paper_conf_icppw_planob21_b200 import Pipeline
    from paper_conf_icppw_planob21_b200 import solve_enforced_waits
    base = C.c4()
    w, th, T, Tc = solve_enforced_waits(base.replace(gain=C.TABLE1_G))
    cfg = base.replace(wait_time=tuple(w))      # as tests/test_gpu_c4.py
    wl = workload_for(cfg)
    over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
    g = run_live(cfg, wl, flags=1, slice_words=1024, **over)
    pb = Pipeline(cfg, wl, flags=1, **over)
    db = torch.from_numpy(wl.db.view("int32")).cuda()
    pb.bind_device(db.data_ptr(), wl.db_len)
    pb.drain()
    lb, _ = pb.latency()
    assert g["stats"]["matches"] == pb.stats()["matches"]
    assert np.array_equal(g["lat"], lb)
    pb.close()
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, 6)
    fns = des.make_stage_fns(cfg, ctx)
    rng = des.stream_ranges(cfg, ctx.n_roots)
    for s in (0, 147):
        lo, hi = rng[s]
        hi2 = min(hi, lo + 20_000)
        r = des.simulate_stream(cfg, fns, lo, hi2)
        # the DES is causal: a root that completes before the prefix's last arrival A does not
        # depend on the roots cut off
        lat = np.asarray(r.lat, dtype=np.int64)
        A = (hi2 - lo) * cfg.interarrival
        ok = (lat >= 0) & (np.arange(hi2 - lo) * cfg.interarrival + lat < A)
        assert ok.sum() > 5_000
        assert np.array_equal(g["lat"][lo:hi2][ok], lat[ok]), s


@pytest.mark.parametrize("db_len,streams", [(6, 2), (64, 4), (1000, 3)])
def test_live_tiny_and_empty_streams(db_len, streams):
    """Degenerate live streams: a DB of one root over two streams (stream 0 has no root and no
    words to push), and streams shorter than a word, a chunk and the halo; bit-exact."""
    cfg = _dna(C.THRESHOLD_SLACK, db_len=db_len, streams=streams).replace(
        dna=dict(db_len=db_len, q_len=64, n_planted=0))
    wl = workload_for(cfg)
    g = run_live(cfg, wl, slice_words=3)
    compare(cfg, g, run_oracle(cfg, wl))
