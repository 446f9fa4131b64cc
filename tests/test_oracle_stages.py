"""Pins for oracle.stages.

Independent checks: Python substring search for S0/S1, hand-worked S2/S3
examples, the planted-match recovery property, iid-gain closed forms,
SplitMix64 published vectors, scipy's Poisson CDF for the gain tables.
"""
import math
import os
import random

import numpy as np
import pytest

from plgen import dna, gaintab
from oracle import stages as S

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ACGT = "ACGT"


def ctx_from_str(db: str, q: str, k: int) -> S.DnaContext:
    enc = {c: i for i, c in enumerate(ACGT)}
    dbw = dna.pack(np.array([enc[c] for c in db], dtype=np.uint8))
    qw = dna.pack(np.array([enc[c] for c in q], dtype=np.uint8))
    return S.DnaContext(dbw, len(db), qw, len(q), k)


def test_pack_roundtrip_and_layout():
    rng = np.random.default_rng(0)
    b = rng.integers(0, 4, size=1000, dtype=np.uint8)
    w = dna.pack(b)
    assert (dna.unpack(w, 1000) == b).all()
    # base j at bits 2*(j mod 16) of word j//16 (DESIGN.md data layout)
    for j in (0, 1, 15, 16, 17, 999):
        assert S.base(w, j) == b[j]
    assert int(w[0]) & 3 == b[0] and (int(w[0]) >> 30) & 3 == b[15]


def test_key_first_base_most_significant():
    ctx = ctx_from_str("ACGTAC" + "A" * 10, "ACGTAC", 6)
    # A=0 C=1 G=2 T=3 -> 0*4^5 + 1*4^4 + 2*4^3 + 3*4^2 + 0*4 + 1 = 256 + 128 + 48 + 1
    assert S.key(ctx.db, 0, 6) == 433


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_s0_s1_vs_substring_search(seed):
    rnd = random.Random(seed)
    k, u = 3, 4
    db = "".join(rnd.choice(ACGT) for _ in range(300))
    q = "".join(rnd.choice(ACGT) for _ in range(80))
    ctx = ctx_from_str(db, q, k)
    for p in range(len(db) - k + 1):
        kmer = db[p:p + k]
        kept = S.s0_seed_lookup(ctx, (p, 0, None))
        assert bool(kept) == (kmer in q)
        # all occurrences of kmer in q by repeated str.find (overlapping)
        occ, i = [], q.find(kmer)
        while i >= 0:
            occ.append(i)
            i = q.find(kmer, i + 1)
        hits = S.s1_hit_enum(ctx, (p, 0, None), u)
        assert hits == [(p, j, occ[j]) for j in range(min(len(occ), u))]


def test_s2_worked_example():
    # k=4 seed "ACGT" at db p=4, query q=4.  Right of the seed (W=4):
    #   db   "AAT..." vs query "AAG..." -> +1 +1 -3  => R = 1, 2, -1, ...; best_right = 2
    # Left (mirror, db[p-1], db[p-2], ...): db "CCCC" reversed vs query "GCCC" reversed:
    #   db[3]='C' q[3]='C' +1; db[2]='C' q[2]='C' +1; db[1]='C' q[1]='C' +1; db[0]='C' q[0]='G' -3
    #   => L = 1, 2, 3, 0; best_left = 3.   k + 3 + 2 = 9.
    db = "CCCC" + "ACGT" + "AATTTTTT"
    q = "GCCC" + "ACGT" + "AAGCCCCC"
    ctx = ctx_from_str(db, q, 4)
    e = (4, 0, 4)
    assert S.s2_window(ctx, e, 4, 9) == [e]
    assert S.s2_window(ctx, e, 4, 10) == []
    # W = 1 limits both sides to one step: k + 1 + 1 = 6
    assert S.s2_window(ctx, e, 1, 6) == [e]
    assert S.s2_window(ctx, e, 1, 7) == []


def test_s2_truncates_at_sequence_ends():
    # seed at the very start of both sequences: no left extension possible
    db = "ACGTA" + "C" * 5
    q = "ACGTA" + "G" * 5
    ctx = ctx_from_str(db, q, 4)
    # right: +1 (A=A) then -3... best_right = 1; left: none -> 4 + 0 + 1 = 5
    assert S.s2_window(ctx, (0, 0, 0), 8, 5) == [(0, 0, 0)]
    assert S.s2_window(ctx, (0, 0, 0), 8, 6) == []


def test_s3_worked_example_xdrop():
    # k=6 seed at p=q=3.  Left: 3 matches then sequence start -> best_left 3, dL 3.
    # Right: 5 matches, then mismatches: score 5 -> 2 -> -1 -> ... after 7 mismatches
    #   5 - 21 = -16 <= best - X = 5 - 20 = -15 -> stop.  best_right 5, dR 5.
    # The trailing matches after the stop are never reached.
    left = "GAT"
    seed = "ACGTAC"
    right_db = "TTTTT" + "AAAAAAA" + "CCCCCCCCCC"
    right_q = "TTTTT" + "GGGGGGG" + "CCCCCCCCCC"
    db = left + seed + right_db
    q = left + seed + right_q
    ctx = ctx_from_str(db, q, 6)
    rec = S.s3_xdrop(ctx, (3, 0, 3), 20, 14)
    assert rec == [(3, 3, 0, 0, 6 + 3 + 5, 14)]
    assert S.s3_xdrop(ctx, (3, 0, 3), 20, 15) == []


def test_s3_smallest_d_attaining_best():
    # right: +1 -3 +1 +1 +1 -> R = 1, -2, -1, 0, 1: best 1 first attained at d = 1
    db = "ACGTAC" + "A" + "C" + "AAA" + "T" * 40
    q = "ACGTAC" + "A" + "G" + "AAA" + "G" * 40
    ctx = ctx_from_str(db, q, 6)
    rec = S.s3_xdrop(ctx, (0, 0, 0), 20, 0)
    assert rec == [(0, 0, 0, 0, 6 + 0 + 1, 7)]


def test_planted_segments_yield_overlapping_hsp():
    """P12: every planted segment of length >= 64 with 5% substitutions yields >= 1 HSP
    overlapping it (T3 = 30, X = 20)."""
    wl = dna.make_dna(5, db_len=1 << 15, q_len=1024, n_planted=8)
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, 6)
    for d_off, q_off, L in wl.planted:
        found = False
        for p in range(d_off, d_off + L - 6 + 1):
            if not S.s0_seed_lookup(ctx, (p, 0, None)):
                continue
            for e in S.s1_hit_enum(ctx, (p, 0, None), 16):
                for rec in S.s3_xdrop(ctx, e, 20, 30):
                    if rec[2] < d_off + L and rec[2] + rec[4] > d_off:
                        found = True
            if found:
                break
        assert found, (d_off, q_off, L)


def test_iid_seed_gain_closed_form():
    """P12: on iid DNA, P(k-mer present in the query) = 1 - (1 - 4^-k)^(Lq-k+1) approx
    (0.2203 for k=6, Lq=1024); sampled over 200k DB positions."""
    wl = dna.make_dna(11, db_len=200_000, q_len=1024, n_planted=0)
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, 6)
    kept = sum(1 for p in range(ctx.n_roots) if S.s0_seed_lookup(ctx, (p, 0, None)))
    g0 = kept / ctx.n_roots
    expect = 1 - (1 - 4.0 ** -6) ** (1024 - 6 + 1)
    assert abs(expect - 0.2203) < 5e-4
    assert abs(g0 - expect) < 0.012


def test_splitmix64_published_vectors():
    with open(os.path.join(GOLD, "splitmix64.txt")) as f:
        rows = [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]
    for n, out in rows:
        n = int(n)
        assert S.splitmix64(((n - 1) * S.SM_GAMMA) % (1 << 64)) == int(out, 16)


def test_bernoulli_and_poisson_tables():
    from scipy.stats import poisson
    assert gaintab.bernoulli_table(0.5)[0] == 1 << 63
    assert gaintab.bernoulli_table(0.0)[0] == 0
    tab = gaintab.poisson_capped_table(1.92, 16)
    for k in range(16):
        assert abs(tab[k] / 2.0 ** 64 - poisson.cdf(k, 1.92)) < 1e-12
    assert all(tab[i] <= tab[i + 1] for i in range(15))


def test_gain_stage_statistics():
    """Bernoulli(g) keeps ~g; min(Poisson(1.92),16) has mean ~1.92 and the Poisson pmf."""
    from scipy.stats import poisson
    thr = gaintab.bernoulli_table(0.379)[0]
    n = 40_000
    kept = sum(1 for r in range(n) if S.g_bernoulli(7, 0, (r, 0, None), thr))
    assert abs(kept / n - 0.379) < 4 * math.sqrt(0.379 * 0.621 / n)
    tab = gaintab.poisson_capped_table(1.92, 16)
    counts = [len(S.g_poisson_capped(7, 1, (r, 0, None), tab, 16)) for r in range(n)]
    mean = sum(counts) / n
    assert abs(mean - 1.92) < 4 * math.sqrt(1.92 / n)
    for k in range(4):
        frac = counts.count(k) / n
        pk = poisson.pmf(k, 1.92)
        assert abs(frac - pk) < 4 * math.sqrt(pk * (1 - pk) / n)
    # children lineage is mixed radix (lin*u + j) and distinct
    ch = S.g_poisson_capped(7, 1, (3, 5, None), [0] * 16, 16)
    assert [c[1] for c in ch] == [5 * 16 + j for j in range(16)]


def test_table1_golden_matches_configs():
    from plgen import configs as C
    with open(os.path.join(GOLD, "table1.txt")) as f:
        rows = [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]
    t = tuple(int(r[1]) for r in rows[:4])
    g = tuple(float(r[2]) for r in rows[:3])
    b = tuple(int(x) for x in rows[4][1:])
    assert t == C.TABLE1_T and g == C.TABLE1_G and b == C.PAPER_B


def test_unpack_bytes_matches_base():
    """The vectorised unpack (the oracle's DB view) gives base() for every position, including
    a ragged last word."""
    import numpy as np
    from plgen import dna as G
    rng = np.random.default_rng(7)
    for n in (1, 15, 16, 17, 1000, 4099):
        codes = rng.integers(0, 4, size=n, dtype=np.uint8)
        words = G.pack(codes)
        ub = S.unpack_bytes(words, n)
        assert len(ub) == n
        assert list(ub) == [S.base(words, j) for j in range(n)] == list(codes)
