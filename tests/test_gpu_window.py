"""GPU parity of the sliding smem DB window (a1).

A stream whose DB range exceeds its smem ring slides the window: chunks are TMA-loaded as
the nodes advance (executor.cu win_step), bounded by the smallest root any node will still
read.  The window is a cache -- reads outside it go to the bound DB -- so every result must be
bit-exact with the oracle whatever the ring size, and a ring much smaller than the stream
must actually refill (pl_stats.window_refills).
"""
import numpy as np
import pytest

from plgen import configs as C
from parity import compare, run_gpu, run_oracle, workload_for

pytestmark = pytest.mark.gpu


def _dna(policy, db_len=1 << 16, streams=2, **kw):
    cfg = C.c2(n_streams=streams, dna=dict(db_len=db_len, q_len=1024, n_planted=16), **kw)
    if policy == C.FIXED_WAIT:
        return cfg.replace(wait_time=(993, 2422, 965, 1628))
    if policy == C.THRESHOLD_SLACK:
        return cfg.replace(policy=policy, wait_threshold=(128, 127, 99, 10))
    return cfg.replace(policy=policy, block_size=2688)


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
@pytest.mark.parametrize("ring,chunk", [(512, 64), (1024, 256)])
def test_sliding_window_logical(policy, ring, chunk):
    """32 K-root streams through an 8 K / 16 K-base ring: many refills, bit-exact results."""
    cfg = _dna(policy)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, window_words=ring, window_chunk_words=chunk)
    assert g["stats"]["window_refills"] > 0
    compare(cfg, g, run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_ring_smaller_than_reach(policy):
    """A ring shorter than one root's extension reach (2 x (q_len + 48) bases): nearly every
    read falls back to the bound DB; results unchanged."""
    cfg = _dna(policy, db_len=1 << 15)
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl, window_words=128, window_chunk_words=64), run_oracle(cfg, wl))


def test_sliding_window_forced_spill():
    """Sliding window and HBM-spilled queues together."""
    cfg = _dna(C.FIXED_WAIT, streams=3)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, window_words=512, window_chunk_words=64, queue_capacity=64)
    assert sum(g["stats"]["spilled"]) > 0 and g["stats"]["window_refills"] > 0
    compare(cfg, g, run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_sliding_window_physical_replay(policy):
    """Physical clock: the firing membership, latencies (units), traces and matches replay the
    oracle's logical schedule while the window slides under real-time pacing."""
    cfg = _dna(policy).replace(clock=C.CLOCK_GLOBALTIMER, ns_per_unit=4.0, interarrival=40,
                               deadline=10**9)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, window_words=1024, window_chunk_words=128)
    assert g["stats"]["window_refills"] > 0
    o = run_oracle(cfg, wl)
    assert g["matches"] == [tuple(m) for m in o.matches]
    assert np.array_equal(g["trace"], np.asarray(o.trace, dtype=np.uint32))
    assert np.array_equal(g["lat"], np.asarray(o.lat, dtype=np.int64))


def test_sliding_window_bind_host():
    """The window refilled by TMA straight from pinned host memory (pl_pipeline_bind_host)."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    cfg = _dna(C.FIXED_WAIT)
    wl = workload_for(cfg)
    host = torch.from_numpy(wl.db.view("int32").copy()).pin_memory()
    pl = Pipeline(cfg, wl, flags=7, window_words=512, window_chunk_words=64)
    pl.bind_host(host.data_ptr(), wl.db_len)
    pl.drain()
    g = dict(stats=pl.stats(), matches=pl.results())
    g["lat"], _ = pl.latency()
    g["trace"] = pl.trace()
    g["firings"] = pl.firings()
    pl.close()
    assert g["stats"]["window_refills"] > 0
    compare(cfg, g, run_oracle(cfg, wl))
