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
