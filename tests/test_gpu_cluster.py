"""GPU parity of N4: every stream on a cluster of N CTAs,
node i on CTA rank i, its input queue in that CTA's shared memory written by node i-1 over
DSMEM (PL_CLUSTER_NODES).  The mapping changes where the nodes run, not what the method
computes: matches, traces, per-root latencies, firing logs and every counter must be bit-exact
with the oracle, as for the one-CTA-per-stream executor -- including HBM spills, a sliding DB
window per CTA, and the physical clock's logical schedule.
"""
import pytest

from plgen import configs as C
from parity import compare, run_gpu, run_oracle, workload_for

pytestmark = pytest.mark.gpu

CL = 32   # PL_CLUSTER_NODES


def _c1(policy, **kw):
    base = C.c1(**kw)
    if policy == C.FIXED_WAIT:
        return base.replace(wait_time=(64, 90))
    return base.replace(policy=policy, wait_threshold=(32, 23))


def _dna(policy, db_len=1 << 16, streams=5, **kw):
    cfg = C.c2(n_streams=streams, dna=dict(db_len=db_len, q_len=1024, n_planted=12), **kw)
    if policy == C.FIXED_WAIT:
        return cfg.replace(wait_time=(993, 2422, 965, 1628))
    return cfg.replace(policy=policy, wait_threshold=(128, 127, 99, 10))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
@pytest.mark.parametrize("streams,X", [(1, 5000), (7, 777)])
def test_cluster_c1_gain_model(policy, streams, X):
    cfg = _c1(policy, n_streams=streams, n_roots=X)
    compare(cfg, run_gpu(cfg, None, flags=7 | CL), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_cluster_blast_gain_model(policy):
    """The 4-stage random-gain BLAST model (Table 1): 4-CTA clusters."""
    from oracle import solver as SV
    tau, D = 10, 50_000
    cfg = C.gain_model_blast(interarrival=tau, deadline=D, n_streams=4, n_roots=6000, seed=3)
    Pc, _ = SV.fig1_continuous(C.TABLE1_T, C.TABLE1_G, C.PAPER_B, 128, tau, D)
    if policy == C.FIXED_WAIT:
        cfg = cfg.replace(wait_time=tuple(int(Pc[i]) - C.TABLE1_T[i] for i in range(4)))
    else:
        P = [int(x) for x in Pc]
        cfg = cfg.replace(policy=policy, wait_threshold=tuple(SV.thresholds(C.TABLE1_G, P, tau, 128)))
    compare(cfg, run_gpu(cfg, None, flags=7 | CL), run_oracle(cfg, None))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_cluster_dna(policy):
    cfg = _dna(policy)
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl, flags=7 | CL), run_oracle(cfg, wl))


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_cluster_dna_forced_spill_and_sliding_window(policy):
    """Tiny smem rings (every edge spills to HBM, read back by another SM through L2) and a
    256-word DB window per CTA sliding behind its own node."""
    cfg = _dna(policy, streams=3)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, flags=7 | CL, queue_capacity=64, window_words=256, window_chunk_words=64)
    assert sum(g["stats"]["spilled"]) > 0 and g["stats"]["window_refills"] > 0
    compare(cfg, g, run_oracle(cfg, wl))


def test_cluster_physical_logical_schedule():
    """%globaltimer clock: the committed schedule is the oracle's (bit-exact), measured
    latencies are positive and bounded by the schedule's plus the measured lateness."""
    cfg = _dna(C.THRESHOLD_SLACK, streams=4).replace(clock=C.CLOCK_GLOBALTIMER, ns_per_unit=1.0,
                                                     service_time=(20_000,) * 4, interarrival=300,
                                                     deadline=10_000_000)
    wl = workload_for(cfg)
    g = run_gpu(cfg, wl, flags=7 | 8 | CL)
    compare(cfg, g, run_oracle(cfg, wl))
    st = g["stats"]
    assert (g["lat_ns"] > 0).all()
    assert (g["lat_ns"] <= g["lat"] + max(st["max_lateness_ns"]) + 64).all()


def test_cluster_rejects_monolithic_and_live():
    from paper_conf_icppw_planob21_b200 import Pipeline
    from paper_conf_icppw_planob21_b200._pl import PlError
    cfg = _dna(C.THRESHOLD_SLACK)
    wl = workload_for(cfg)
    with pytest.raises(PlError):
        Pipeline(cfg.replace(policy=C.MONOLITHIC, block_size=2688), wl, flags=CL)
    pl = Pipeline(cfg, wl, flags=CL)
    with pytest.raises(PlError):
        pl.live_start()
    pl.close()


@pytest.mark.parametrize("policy", [C.FIXED_WAIT, C.THRESHOLD_SLACK])
def test_cluster_eight_nodes(policy):
    """N = 8: clusters of 8 CTAs (the portable maximum), one random-gain node per CTA."""
    st = [C.Stage(C.BERNOULLI, 0.8, 1), C.Stage(C.POISSON_CAPPED, 1.3, 4), C.Stage(C.BERNOULLI, 0.6, 1),
          C.Stage(C.FIXED_GAIN, 2.0, 2), C.Stage(C.BERNOULLI, 0.5, 1), C.Stage(C.KEEP_EVERY, 3.0, 1),
          C.Stage(C.POISSON_CAPPED, 0.9, 3), C.Stage(C.BERNOULLI, 0.7, 1)]
    cfg = C.Config(name="n8", stages=st, service_time=(40, 55, 30, 45, 25, 35, 50, 20), vector_width=128,
                   deadline=20_000, interarrival=3, b=(1,) * 8, wait_time=(300, 100, 50, 80, 40, 60, 90, 30),
                   wait_threshold=(64, 32, 16, 16, 8, 8, 4, 4), policy=policy, n_streams=3, n_roots=3000, seed=5)
    compare(cfg, run_gpu(cfg, None, flags=7 | CL), run_oracle(cfg, None))


@pytest.mark.parametrize("v", [32, 256])
def test_cluster_vector_widths(v):
    cfg = _dna(C.THRESHOLD_SLACK, db_len=1 << 15, streams=3).replace(vector_width=v,
                                                                     wait_threshold=(v, v - 1, v // 2, 4))
    wl = workload_for(cfg)
    compare(cfg, run_gpu(cfg, wl, flags=7 | CL), run_oracle(cfg, wl))


def test_cluster_poisson_arrivals():
    from plgen import arrivals as A
    cfg = _dna(C.THRESHOLD_SLACK, db_len=1 << 15, streams=3)
    wl = workload_for(cfg)
    arr = A.poisson(3, A.stream_sizes(wl.db_len - 6 + 1, cfg.n_streams), cfg.interarrival)
    compare(cfg, run_gpu(cfg, wl, flags=7 | CL, arrivals=arr), run_oracle(cfg, wl, arrivals=arr))
