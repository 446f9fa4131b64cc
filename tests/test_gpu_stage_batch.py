"""Per-stage batch kernels (pl_stage_batch, SURVEY K-BENCH) vs the oracle's stage functions:
S0 -> S1 -> S2 -> S3 over every root of a DNA workload, outputs compared as multisets (the
batch kernel keeps order only within a vector).  Independent of the scheduler."""
import numpy as np
import pytest

from plgen import configs as C
from parity import workload_for

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("db_len,heavy", [(1 << 16, False), (40_003, False), (1 << 18, True), (1 << 20, True)])
def test_stage_chain_matches_oracle(db_len, heavy):
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    from oracle import stages as S
    dna = dict(db_len=db_len, q_len=1024, n_planted=12)
    if heavy:   # c4's recipe (repeat islands, tandem-repeat query motifs) at a size the oracle runs
        dna.update(heavy_tailed=True)
    cfg = C.c2(n_streams=1, dna=dna, wait_time=(0, 0, 0, 0))
    wl = workload_for(cfg)
    pl = Pipeline(cfg, wl, flags=0)
    pl.push(wl.db, wl.db_len)
    R = db_len - 6 + 1
    bufs = [torch.empty((R * 16, 2), dtype=torch.int32, device="cuda") for _ in range(2)]
    n0, _ = pl.stage_batch(0, 0, R, 0, bufs[0].data_ptr(), R * 16)
    n1, _ = pl.stage_batch(1, bufs[0].data_ptr(), n0, 0, bufs[1].data_ptr(), R * 16)
    s1 = bufs[1][:n1].cpu().numpy().astype(np.uint32)
    n2, _ = pl.stage_batch(2, bufs[1].data_ptr(), n1, 0, bufs[0].data_ptr(), R * 16)
    s2 = bufs[0][:n2].cpu().numpy().astype(np.uint32)
    n3, _ = pl.stage_batch(3, bufs[0].data_ptr(), n2, 0, 0, 0)
    matches = pl.results()
    pl.close()
    # oracle, stage by stage
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, 6)
    o0 = [(p, 0, None) for p in range(R) if S.s0_seed_lookup(ctx, (p, 0, None))]
    o1 = [h for e in o0 for h in S.s1_hit_enum(ctx, e, 16)]
    o2 = [h for e in o1 for h in S.s2_window(ctx, e, 8, 9)]
    o3 = sorted(m for e in o2 for m in S.s3_xdrop(ctx, e, 20, 30))
    assert n0 == len(o0)
    assert sorted((int(a), int(b) & 0xffff, int(b) >> 16) for a, b in s1) == sorted((p, q, j) for p, j, q in o1)
    assert sorted((int(a), int(b) & 0xffff) for a, b in s2) == sorted((p, q) for p, j, q in o2)
    assert n3 == len(o3) and matches == o3


def _gain_chain(cfg, n_roots):
    """Every stage of a random-gain pipeline through pl_stage_batch (root lineage carried in
    entry.y), vs the oracle's per-item stage functions (oracle.des.make_stage_fns) on the same
    seeded hashes; outputs compared as multisets of (root, lineage)."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    from oracle import des
    pl = Pipeline(cfg, None, flags=0)
    pl.push(None, n_roots)
    cap = n_roots * 32
    bufs = [torch.empty((cap, 2), dtype=torch.int32, device="cuda") for _ in range(2)]
    fns = des.make_stage_fns(cfg, None)
    ref = [(r, 0, None) for r in range(n_roots)]
    n_in, src = n_roots, 0
    for st in range(cfg.n_stages):
        last = st + 1 == cfg.n_stages
        dst = 0 if last else bufs[st % 2].data_ptr()
        n_out, _ = pl.stage_batch(st, src, n_in, 0, dst, 0 if last else cap)
        ref = [o for e in ref for o in fns[st](e)]
        assert n_out == len(ref), f"stage {st}: {n_out} outputs, oracle {len(ref)}"
        if not last:
            got = bufs[st % 2][:n_out].cpu().numpy().astype(np.uint32)
            assert sorted((int(a), int(b)) for a, b in got) == sorted((r, l) for r, l, _ in ref), f"stage {st}"
        n_in, src = n_out, dst
    pl.close()


@pytest.mark.parametrize("n_roots", [1, 127, 4099, 50_000])
def test_stage_chain_gain_model_blast(n_roots):
    """Table 1's random-gain model: Bernoulli -> min(Poisson(1.92), 16) -> Bernoulli -> Bernoulli(1)."""
    _gain_chain(C.gain_model_blast(n_roots=n_roots), n_roots)


def test_stage_chain_c1_and_keep_every():
    """c1 (Bernoulli 0.5 -> fixed gain 2) and c1r (keep every 2nd -> fixed gain 2), ragged tails."""
    _gain_chain(C.c1(n_roots=10_007), 10_007)
    _gain_chain(C.c1r(n_roots=333), 333)


@pytest.mark.parametrize("first_root", [0, 64, 37, 1 << 12])
def test_s0_first_root_paths(first_root):
    """S0 through pl_stage_batch from an arbitrary first root: the rolling-k-mer path (first_root a
    multiple of 64) and the per-item path (otherwise) both equal the oracle's S0 on every root, in
    root order (the kernel keeps input order within a warp's chunk; chunks are sorted here)."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    from oracle import stages as S
    cfg = C.c2(n_streams=1, dna=dict(db_len=40_003, q_len=1024, n_planted=12, heavy_tailed=True),
               wait_time=(0, 0, 0, 0))
    wl = workload_for(cfg)
    pl = Pipeline(cfg, wl, flags=0)
    pl.push(wl.db, wl.db_len)
    R = wl.db_len - 6 + 1
    n = R - first_root
    buf = torch.empty((n + 64, 2), dtype=torch.int32, device="cuda")
    n0, _ = pl.stage_batch(0, 0, n, first_root, buf.data_ptr(), n + 64)
    got = buf[:n0].cpu().numpy().astype(np.uint32)
    pl.close()
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, 6)
    ref = [p for p in range(first_root, R) if S.s0_seed_lookup(ctx, (p, 0, None))]
    assert n0 == len(ref)
    assert sorted(int(a) for a, _ in got) == ref and all(int(b) == 0 for _, b in got)


def test_s0_roots_past_db_end_rejected():
    """pl_stage_batch refuses stage-0 roots beyond the DB's last k-mer (PL_EINVAL), which would
    otherwise read k-mers of the zero padding."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    from paper_conf_icppw_planob21_b200._pl import PlError
    cfg = C.c2(n_streams=1, dna=dict(db_len=1 << 14, q_len=1024, n_planted=4), wait_time=(0, 0, 0, 0))
    wl = workload_for(cfg)
    pl = Pipeline(cfg, wl, flags=0)
    pl.push(wl.db, wl.db_len)
    R = wl.db_len - 6 + 1
    buf = torch.empty((R + 64, 2), dtype=torch.int32, device="cuda")
    n_ok, _ = pl.stage_batch(0, 0, R, 0, buf.data_ptr(), R + 64)
    with pytest.raises(PlError):
        pl.stage_batch(0, 0, R, 1, buf.data_ptr(), R + 64)
    pl.close()
    assert n_ok >= 0
