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
