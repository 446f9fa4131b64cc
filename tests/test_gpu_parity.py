"""GPU parity: the CUDA path (C-ABI, logical clock) vs the oracle, bit-exact.

Covers every policy (FIXED_WAIT, THRESHOLD_SLACK, MONOLITHIC), both stage
families (random-gain model of PAPER.md L210 and the BLAST-style DNA chain),
multi-stream grids, ragged stream tails, empty streams, and forced HBM spills.
"""
import pytest

from plgen import configs as C
from oracle import solver as SV
from parity import compare, run_gpu, run_oracle, workload_for

pytestmark = pytest.mark.gpu


def _c1(policy, **kw):
    base = C.c1(**kw)
    if policy == C.FIXED_WAIT:
        return base.replace(wait_time=(64, 90))
    if policy == C.THRESHOLD_SLACK:
        return base.replace(policy=policy, wait_threshold=(32, 23))
    return base.replace(policy=policy, block_size=64)


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
@pytest.mark.parametrize("streams,X", [(1, 5000), (3, 3001), (7, 777)])
def test_c1_gain_model(policy, streams, X):
    cfg = _c1(policy, n_streams=streams, n_roots=X)
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_c1_full_size(policy):
    """BASELINE configs[0] at full size: 1e5 items, v = 32."""
    cfg = _c1(policy)
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
@pytest.mark.parametrize("tau,D", [(10, 50_000), (100, 25_000)])
def test_blast_gain_model(policy, tau, D):
    """The paper-faithful random-gain BLAST model (Table 1): Bernoulli / censored Poisson."""
    cfg = C.gain_model_blast(interarrival=tau, deadline=D, n_streams=4, n_roots=6000, seed=3)
    if policy == C.FIXED_WAIT:
        Pc, _ = SV.fig1_continuous(C.TABLE1_T, C.TABLE1_G, C.PAPER_B, 128, tau, D)
        cfg = cfg.replace(wait_time=tuple(int(Pc[i]) - C.TABLE1_T[i] for i in range(4)))
    elif policy == C.THRESHOLD_SLACK:
        Pc, _ = SV.fig1_continuous(C.TABLE1_T, C.TABLE1_G, C.PAPER_B, 128, tau, D)
        P = [int(x) for x in Pc]
        cfg = cfg.replace(policy=policy, wait_threshold=tuple(SV.thresholds(C.TABLE1_G, P, tau, 128)))
    else:
        M, _ = SV.fig2_exhaustive(C.TABLE1_T, C.TABLE1_G, 128, tau, D)
        cfg = cfg.replace(policy=policy, block_size=M)
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


def _dna(policy, db_len=1 << 16, streams=5, **kw):
    cfg = C.c2(n_streams=streams, dna=dict(db_len=db_len, q_len=1024, n_planted=12), **kw)
    if policy == C.FIXED_WAIT:
        return cfg.replace(wait_time=(993, 2422, 965, 1628))
    if policy == C.THRESHOLD_SLACK:
        return cfg.replace(policy=policy, wait_threshold=(128, 127, 99, 10))
    return cfg.replace(policy=policy, block_size=2688)


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_dna_pipeline_small(policy):
    cfg = _dna(policy)
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl), run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_dna_forced_spill(policy):
    """Tiny smem rings: every edge overflows into the HBM ring; results must not change."""
    cfg = _dna(policy, streams=3)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, queue_capacity=64)
    assert sum(g["stats"]["spilled"]) > 0
    compare(cfg, g, run_oracle(cfg, wl))


def test_more_streams_than_roots():
    cfg = _c1(C.FIXED_WAIT, n_streams=9, n_roots=0)
    g = run_gpu(cfg, None, flags=0)
    assert g["stats"]["roots"] == 0 and g["stats"]["errors"] == 0


def test_ragged_streams_dna():
    """Streams whose lengths differ by one root and a DB length that is not a multiple of 16."""
    cfg = _dna(C.FIXED_WAIT, db_len=40_003, streams=6)
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl), run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
@pytest.mark.parametrize("v", [32, 64, 256])
def test_vector_widths_dna(policy, v):
    """v = 32..256 lanes per node (one warp group each; v = 256 -> 1024 threads, N = 4)."""
    cfg = _dna(policy, db_len=1 << 15, streams=3).replace(vector_width=v)
    if policy == C.THRESHOLD_SLACK:
        cfg = cfg.replace(wait_threshold=tuple(min(t, v) for t in cfg.wait_threshold))
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl), run_oracle(cfg, wl))


def test_threshold_slack_guard():
    """THRESHOLD_SLACK with a slack guard added to every R_i (both sides)."""
    cfg = _dna(C.THRESHOLD_SLACK, db_len=1 << 15, streams=3).replace(slack_guard=7000)
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl), run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_eight_node_gain_pipeline(policy):
    """N = 8 random-gain nodes (the ABI maximum), v = 128 -> 1024 threads."""
    st = [C.Stage(C.BERNOULLI, 0.8, 1), C.Stage(C.POISSON_CAPPED, 1.3, 4), C.Stage(C.BERNOULLI, 0.6, 1),
          C.Stage(C.FIXED_GAIN, 2.0, 2), C.Stage(C.BERNOULLI, 0.5, 1), C.Stage(C.KEEP_EVERY, 3.0, 1),
          C.Stage(C.POISSON_CAPPED, 0.9, 3), C.Stage(C.BERNOULLI, 0.7, 1)]
    cfg = C.Config(name="n8", stages=st, service_time=(40, 55, 30, 45, 25, 35, 50, 20), vector_width=128,
                   deadline=20_000, interarrival=3, b=(1,) * 8, wait_time=(300, 100, 50, 80, 40, 60, 90, 30),
                   wait_threshold=(64, 32, 16, 16, 8, 8, 4, 4), policy=policy, n_streams=3, n_roots=3000, seed=5)
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_physical_other_policies_replay(policy):
    """THRESHOLD_SLACK and MONOLITHIC under the %globaltimer clock commit the logical schedule."""
    cfg = _dna(policy, db_len=1 << 15, streams=3).replace(
        clock=C.CLOCK_GLOBALTIMER, ns_per_unit=1.0, service_time=(20_000,) * 4, interarrival=400,
        deadline=10**7, wait_threshold=(64, 32, 16, 8), block_size=1024)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl)
    compare(cfg, g, run_oracle(cfg, wl))
    assert (g["lat_ns"] > 0).all()


def test_bind_host_tma_matches_push():
    """pl_pipeline_bind_host: CTAs stage the DB straight from pinned host memory by TMA;
    results are identical to the pushed (H2D-copied) DB and to the oracle."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    cfg = _dna(C.FIXED_WAIT, db_len=1 << 16, streams=5)
    wl = workload_for(cfg)
    host = torch.from_numpy(wl.db.view("int32")).pin_memory()
    pl = Pipeline(cfg, wl, flags=7)
    pl.bind_host(host.data_ptr(), wl.db_len)
    pl.drain()
    g = dict(stats=pl.stats(), matches=pl.results(), firings=pl.firings(), trace=pl.trace())
    g["lat"], g["lat_ns"] = pl.latency()
    summ = pl.summary()
    pl.close()
    o = run_oracle(cfg, wl)
    compare(cfg, g, o)
    assert summ["roots"] == g["stats"]["roots"] and summ["matches"] == len(o.matches)
    assert summ["max_latency"] == max(o.lat) and summ["miss_events"] == g["stats"]["miss_events"]


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_poisson_arrivals_gain_model(policy):
    """N2: Poisson arrivals given as per-root arrival times."""
    from plgen import arrivals as A
    cfg = _c1(policy, n_streams=4, n_roots=3000)
    arr = A.poisson(9, A.stream_sizes(cfg.n_roots * cfg.n_streams, cfg.n_streams), cfg.interarrival)
    g = run_gpu(cfg, None, arrivals=arr)
    compare(cfg, g, run_oracle(cfg, None, arrivals=arr))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC])
def test_poisson_arrivals_dna(policy):
    from plgen import arrivals as A
    cfg = _dna(policy, db_len=1 << 15, streams=3)
    wl = workload_for(cfg)
    arr = A.poisson(3, A.stream_sizes(wl.db_len - 6 + 1, cfg.n_streams), cfg.interarrival)
    g = run_gpu(cfg, wl, arrivals=arr)
    compare(cfg, g, run_oracle(cfg, wl, arrivals=arr))


# ---------------------------------------------------------------- end of stream (R-DRAIN)

@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
@pytest.mark.parametrize("streams,X", [(1, 5000), (3, 3001), (7, 777)])
def test_eager_drain_gain_model(policy, streams, X):
    cfg = _c1(policy, n_streams=streams, n_roots=X).replace(eager_drain=True)
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_eager_drain_blast_gain_model(policy):
    tau, D = 10, 50_000
    cfg = C.gain_model_blast(interarrival=tau, deadline=D, n_streams=4, n_roots=6000, seed=3, eager_drain=True)
    Pc, _ = SV.fig1_continuous(C.TABLE1_T, C.TABLE1_G, C.PAPER_B, 128, tau, D)
    if policy == C.FIXED_WAIT:
        cfg = cfg.replace(wait_time=tuple(int(Pc[i]) - C.TABLE1_T[i] for i in range(4)))
    else:
        cfg = cfg.replace(policy=policy, wait_threshold=tuple(SV.thresholds(C.TABLE1_G, [int(x) for x in Pc], tau, 128)))
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_eager_drain_dna(policy):
    cfg = _dna(policy).replace(eager_drain=True)
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl), run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_eager_drain_dna_forced_spill(policy):
    cfg = _dna(policy, streams=3).replace(eager_drain=True)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, queue_capacity=64)
    assert sum(g["stats"]["spilled"]) > 0
    compare(cfg, g, run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_eager_drain_poisson(policy):
    from plgen import arrivals as A
    cfg = _c1(policy, n_streams=4, n_roots=3000).replace(eager_drain=True)
    arr = A.poisson(11, A.stream_sizes(cfg.n_roots * cfg.n_streams, cfg.n_streams), cfg.interarrival)
    compare(cfg, run_gpu(cfg, None, arrivals=arr), run_oracle(cfg, None, arrivals=arr))


def test_eager_drain_eight_nodes():
    st = [C.Stage(C.BERNOULLI, 0.8, 1), C.Stage(C.POISSON_CAPPED, 1.3, 4), C.Stage(C.BERNOULLI, 0.6, 1),
          C.Stage(C.FIXED_GAIN, 2.0, 2), C.Stage(C.BERNOULLI, 0.5, 1), C.Stage(C.KEEP_EVERY, 3.0, 1),
          C.Stage(C.POISSON_CAPPED, 0.9, 3), C.Stage(C.BERNOULLI, 0.7, 1)]
    cfg = C.Config(name="n8e", stages=st, service_time=(40, 55, 30, 45, 25, 35, 50, 20), vector_width=128,
                   deadline=20_000, interarrival=3, b=(1,) * 8, wait_time=(300, 100, 50, 80, 40, 60, 90, 30),
                   n_streams=3, n_roots=3000, seed=5, eager_drain=True)
    compare(cfg, run_gpu(cfg, None), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_eager_drain_physical_replay(policy):
    """Under %globaltimer the drain commits the logical schedule and shortens the run."""
    cfg = _dna(policy, db_len=1 << 15, streams=3).replace(
        clock=C.CLOCK_GLOBALTIMER, ns_per_unit=1.0, service_time=(20_000,) * 4, interarrival=400,
        deadline=10**7, wait_time=(31_200, 60_000, 80_000, 100_000), wait_threshold=(64, 32, 16, 8), eager_drain=True)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl)
    compare(cfg, g, run_oracle(cfg, wl))
    assert (g["lat_ns"] > 0).all()


def test_repeated_launches_summary_double_buffer():
    """The run summary and match count are double-buffered on the device (each launch zeroes
    the slot of the next one, so no per-launch memset): back-to-back launches without reads
    in between, then reads after each launch, all give the oracle's counts and matches."""
    from paper_conf_icppw_planob21_b200 import Pipeline
    cfg = _dna(C.FIXED_WAIT, db_len=1 << 16, streams=5)
    wl = workload_for(cfg)
    o = run_oracle(cfg, wl)
    pl = Pipeline(cfg, wl, flags=0)
    pl.push(wl.db, wl.db_len)
    for _ in range(3):                   # unread launches: each must start from a zero slot
        pl.launch()
    first = None
    for k in range(4):
        pl.launch()
        s = pl.summary()
        first = first or s
        assert s["roots"] == sum(hi - lo for lo, hi in _ranges(cfg, wl)), k
        assert s["matches"] == len(o.matches), k
        assert s["max_latency"] == max(o.lat) and s["miss_events"] == first["miss_events"], k
        assert pl.results() == [tuple(m) for m in o.matches], k
    st = pl.stats()
    pl.close()
    assert st["launches"] == 7 and st["matches"] == len(o.matches)


def _ranges(cfg, wl):
    from oracle import des
    k = cfg.stages[0].iparam[0]
    return des.stream_ranges(cfg, wl.db_len - k + 1)


def test_physical_loop_time_reported():
    """pl_stats.max_loop_ns (a firing's start to the node's next decision: the real per-firing
    service time incl. publish and bookkeeping) is measured in the physical clock, bounds
    the firing time, and is zero in the logical clock."""
    from paper_conf_icppw_planob21_b200 import Pipeline
    cfg = _dna(C.FIXED_WAIT, db_len=1 << 16, streams=4)
    wl = workload_for(cfg)
    out = {}
    for clock in (0, 1):
        c = cfg.replace(clock=clock, ns_per_unit=1.0, service_time=(4000, 8000, 8000, 20000), interarrival=100,
                        deadline=10 ** 7, wait_time=(100, 100, 100, 100))
        pl = Pipeline(c, wl, flags=0)
        pl.push(wl.db, wl.db_len)
        pl.drain()
        out[clock] = pl.stats()
        pl.close()
    assert all(x == 0 for x in out[0]["max_loop_ns"][:4])
    ph = out[1]
    # node 0 never waits for upstream, so every firing is a sample and the cycle contains it
    assert ph["max_loop_ns"][0] >= ph["max_fire_ns"][0] > 0
    assert all(x >= 0 for x in ph["max_loop_ns"][:4])


def test_pipelined_steps_match_oracle():
    """pl_pipeline_step: run k executes while the host reads run k-1's summary (pinned
    buffers by step parity, copy ordered before the next launch reuses the device slot).
    Every step's summary equals the oracle's counts, from the bound host DB (bind_host TMA)."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    cfg = _dna(C.FIXED_WAIT, db_len=1 << 16, streams=5)
    wl = workload_for(cfg)
    o = run_oracle(cfg, wl)
    roots = sum(hi - lo for lo, hi in _ranges(cfg, wl))
    host = torch.from_numpy(wl.db.view("int32")).pin_memory()
    pl = Pipeline(cfg, wl, flags=0)
    pl.bind_host(host.data_ptr(), wl.db_len)
    got = []
    assert pl.step() is None             # first step: nothing to return yet
    for _ in range(5):
        got.append(pl.step())
    got.append(pl.step_finish())
    assert pl.step_finish() is None
    assert [g["launches"] for g in got] == list(range(1, 7))
    for g in got:
        assert g["roots"] == roots and g["matches"] == len(o.matches)
        assert g["max_latency"] == max(o.lat) and g["errors"] == 0
    s = pl.summary()                     # the synchronous read agrees with the last step
    assert s["roots"] == roots and s["matches"] == len(o.matches)
    assert pl.results() == [tuple(m) for m in o.matches]
    pl.close()


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_extreme_gain_tables(policy):
    """Threshold tables at their edges (the round-1 advisor's prob_to_u64 case): min(Poisson(60), 16)
    -- every CDF(k < 16) is below 2^-64, so every threshold is 0 and every input emits 16 --
    a Bernoulli(1e-30) filter that keeps nothing, and Bernoulli(1.0) that keeps everything."""
    st = [C.Stage(C.BERNOULLI, 1.0, 1), C.Stage(C.POISSON_CAPPED, 60.0, 16), C.Stage(C.BERNOULLI, 1e-30, 1)]
    cfg = C.Config(name="edge", stages=st, service_time=(40, 55, 30), vector_width=32, deadline=50_000,
                   interarrival=20, b=(1, 1, 1), wait_time=(60, 20, 300), wait_threshold=(32, 16, 32),
                   policy=policy, n_streams=2, n_roots=400, seed=9)
    g = run_gpu(cfg, None)
    compare(cfg, g, run_oracle(cfg, None))
    st_ = g["stats"]
    assert st_["produced"][0] == st_["consumed"][0]                 # Bernoulli(1.0) keeps all
    assert st_["produced"][1] == 16 * st_["consumed"][1]            # Poisson(60) capped at 16
    assert st_["produced"][2] == 0                                  # Bernoulli(1e-30) keeps nothing


@pytest.mark.parametrize("k,W,X,u", [(7, 8, 20, 16), (4, 12, 8, 5), (5, 8, 35, 16)])
def test_dna_stage_parameters(k, W, X, u):
    """The DNA chain off its defaults: k = 7 (the largest direct-address table, 16 K entries),
    short seeds with a W = 12 window (the checked S2 walk: W > 8) and a small hit cap u = 5, a
    large X-drop; a query and DB whose lengths are not multiples of 16; bit-exact."""
    stages = C.dna_stages(k=k, u=u, W=W, X=X, T3=max(2 * k, 20))
    cfg = C.c2(stages=stages, n_streams=3, dna=dict(db_len=20_011, q_len=3_001, n_planted=10)).replace(
        policy=C.THRESHOLD_SLACK, wait_threshold=(128, 100, 64, 8))
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl), run_oracle(cfg, wl))
