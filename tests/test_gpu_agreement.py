"""The north_star's physical criterion, on the bench's workload and kernel: per-item latency and
processor utilisation agree with the oracle's logical-clock prediction within 5 % relative.

Configuration: c4 (BASELINE configs[3], the bench's workload) at full size -- 148 streams x
708 K roots, the sliding smem window -- on the %globaltimer clock, THRESHOLD_SLACK (the bench's
headline policy) with PL_FIXED_SERVICE (time-triggered delivery at start + t_i, L69) and
budgets measured at a 1/N processor share, as bench.py does.  Reading R-AGREE:
|measured - logical latency| <= 5 % of the logical latency + 64 ns (two %globaltimer ticks)
for EVERY terminal item.  A run that meets one of the platform's ~1.6 ms SM stalls
(R-STALL; realtime.stalled) is repeated -- the stall is not the executor's -- up to 4 times.

* the bench kernel (no per-item records): the device counts the items outside the band;
* the recording kernel: every root's measured latency (lat_ns) against its logical latency
  (lat, in ns), element by element, plus the logical schedule of sampled streams against the
  oracle's DES bit-exactly.
"""
import numpy as np
import pytest

from plgen import configs as C
from parity import oracle_firings, workload_for

pytestmark = pytest.mark.gpu

D, SG = 3_500_000, 2_700_000        # bench.py's c4 defaults (R-STALL)
GAINS = (0.04995, 8.9465, 0.56093)       # measured on c4 (realtime.measure_gains)
SAMPLE_STREAMS = (0, 77, 147)
PREFIX = 120_000


@pytest.fixture(scope="module")
def c4():
    import torch
    from paper_conf_icppw_planob21_b200 import realtime
    base = C.c4()
    wl = workload_for(base)
    db = torch.from_numpy(wl.db.view("int32")).cuda()
    over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
    return base, wl, db, over


def _cfg(base, budgets, tau):
    from paper_conf_icppw_planob21_b200 import realtime
    cfg = _cfg_base(base, budgets)
    w, th, T = realtime.solve_at(cfg.replace(deadline=D - SG), tau)
    return cfg.replace(interarrival=tau, wait_time=tuple(w), wait_threshold=tuple(th))


def _multiset_digest(rows):
    """An order-independent digest of match records: the sum (mod 2^64) of a per-record hash."""
    r = rows.astype(np.uint64)
    h = np.zeros(len(r), dtype=np.uint64)
    for j, k in enumerate((0x9E3779B97F4A7C15, 0xBF58476D1CE4E5B9, 0x94D049BB133111EB, 0xD6E8FEB86659FD93,
                           0xA0761D6478BD642F, 0xE7037ED1A0B428DB)):
        h = (h ^ r[:, j]) * np.uint64(k)
        h ^= h >> np.uint64(29)
    return int(h.sum(dtype=np.uint64)), len(r)


def _run_unstalled(cfg, wl, db, over, flags, tries=4):
    from paper_conf_icppw_planob21_b200 import Pipeline, realtime
    seen = []
    for _ in range(tries):
        pl = Pipeline(cfg, wl, flags=flags, **over)
        pl.bind_device(db.data_ptr(), wl.db_len)
        pl.drain()
        st = pl.stats()
        out = {"stats": st}
        if flags & 1:
            out["lat"], out["lat_ns"] = pl.latency()
        if flags & 4:
            out["firings"] = pl.firings()
        out["digest"] = _multiset_digest(pl.results_raw())
        pl.close()
        if not realtime.stalled(st):
            return out
        seen.append(st["max_lateness_ns"])
    pytest.skip(f"every run met a platform stall (per-node lateness of each run: {seen})")


def _tau(base, b):
    """1.5 x the node-3 island bound u t_3 / v, and at least 1.3 x the smallest Fig. 1-feasible tau0."""
    from paper_conf_icppw_planob21_b200 import realtime
    cfg = _cfg_base(base, b)
    t_min = realtime.min_feasible_tau(cfg.replace(deadline=D - SG))
    assert t_min is not None, b
    return max(int(1.5 * 16 * b[3] / 128), int(1.3 * t_min))


def _cfg_base(base, budgets):
    return base.replace(clock=C.CLOCK_GLOBALTIMER, ns_per_unit=1.0, service_time=budgets, gain=GAINS, deadline=D,
                        b=C.PAPER_B, policy=C.THRESHOLD_SLACK, slack_guard=max(budgets) + SG)


def _budgets(c4, flags):
    from paper_conf_icppw_planob21_b200 import realtime
    base, wl, db, over = c4
    b, _ = realtime.calibrate_budgets(base, wl, db.data_ptr(), over=over, probe_t=1000, probe_tau=20, margin=1.1,
                                      slack_ns=128, flags=flags)
    return b


def test_bench_kernel_every_item_within_5pct(c4):
    """The record-free kernel bench.py times, at 1.5 x the node-3 island bound u t_3 / v."""
    from paper_conf_icppw_planob21_b200._pl import PL_FIXED_SERVICE
    base, wl, db, over = c4
    b = _budgets(c4, 0)                 # bench.py calibrates with the record-free kernel, flags 0
    tau = _tau(base, b)
    g = _run_unstalled(_cfg(base, b, tau), wl, db, over, PL_FIXED_SERVICE)
    st = g["stats"]
    print("budgets", b, "tau0", tau, "lateness", st["max_lateness_ns"], "rel err max", st["latency_rel_err_max"])
    assert st["roots"] == wl.db_len - 5
    assert st["miss_events_ns"] == 0 and st["miss_events"] == 0 and st["errors"] == 0
    assert st["latency_outliers"] == 0
    # processor utilisation: measured occupancy vs the logical schedule's t_i per firing
    model_busy = sum(st["firings"][i] * b[i] for i in range(4))
    assert abs(sum(st["busy_ns"]) / model_busy - 1) < 0.05
    # the match set and per-node counts are pure functions of the data (R-S0..R-S3): the bench
    # kernel's equal a logical-clock run's (whose schedule tests/test_gpu_c4.py checks vs the oracle)
    from paper_conf_icppw_planob21_b200 import Pipeline
    lg = Pipeline(base.replace(wait_time=(993, 2422, 965, 1628)), wl, **over)
    lg.bind_device(db.data_ptr(), wl.db_len)
    lg.drain()
    sl = lg.stats()
    dl = _multiset_digest(lg.results_raw())
    lg.close()
    assert g["digest"] == dl and st["matches"] == sl["matches"] > 0
    assert st["consumed"] == sl["consumed"] and st["produced"] == sl["produced"]


@pytest.fixture(scope="module")
def c4q():
    """c4's shape (148 streams, heavy-tailed islands, 1 kbp query) at a quarter of its length, so
    that one run (~0.5 s) usually misses the platform's ~1.6 ms SM stalls (every 2-3 s)."""
    import torch
    base = C.c4(dna=dict(db_len=25 << 20, q_len=1024, n_planted=1600, heavy_tailed=True))
    wl = workload_for(base)
    db = torch.from_numpy(wl.db.view("int32")).cuda()
    return base, wl, db, dict(match_capacity=1 << 24, spill_capacity=1 << 19)


def test_recording_kernel_per_root_and_sampled_streams(c4q):
    """Every root's measured latency against its logical one, element by element; the logical
    schedule of sampled streams against the oracle's DES."""
    from oracle import des
    from oracle import stages as S
    base, wl, db, over = c4q
    b = _budgets(c4q, 1)                # the recording kernel's own firing times
    tau = _tau(base, b)
    cfg = _cfg(base, b, tau)
    g = _run_unstalled(cfg, wl, db, over, 1 | 8, tries=8)   # per-root latencies, time-triggered delivery
    st = g["stats"]
    assert st["miss_events_ns"] == 0 and st["errors"] == 0
    lu = g["lat"].astype(np.float64)            # units = ns
    ln = g["lat_ns"].astype(np.float64)
    done = lu >= 0
    assert (ln[done] > 0).all() and (ln[~done] < 0).all()
    err = np.abs(ln[done] - lu[done])
    bad = err > 0.05 * lu[done] + 64
    print("roots", done.sum(), "outside 5%:", int(bad.sum()), "max rel", float((err / lu[done]).max()))
    assert not bad.any()
    assert int(bad.sum()) == st["latency_outliers"]
    # the logical schedule (what the physical run replays) of sampled streams, bit-exact
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, 6)
    fns = des.make_stage_fns(cfg, ctx)
    rng = des.stream_ranges(cfg, ctx.n_roots)
    for s in SAMPLE_STREAMS:
        lo, hi = rng[s]
        hi2 = min(hi, lo + PREFIX)               # the stream's head: the oracle runs it in seconds
        r = des.simulate_stream(cfg, fns, lo, hi2)
        # the DES is causal: its events before the prefix's end A = (hi2 - lo) tau0 do not depend
        # on the roots cut off, so every root that completes before A -- a(r) + D < A -- matches
        n = hi2 - lo if hi2 == hi else max(0, ((hi2 - lo) * tau - D) // tau)
        assert n > 10_000
        assert np.array_equal(g["lat"][lo:lo + n], np.asarray(r.lat[:n], dtype=np.int64)), s
